"""Host-side pin of the kb1_v10 PADU layout choice (csrc/kb1_v10.cuh, OPT bit 7; DESIGN.md §10 `v10.wu`).

The bank model (tools/v10_stageB_bank_model.py) counts shared-memory wavefronts of the k = 4 forward stage B
stores, the stage C loads of UX and the point warps' loads of U / UE, for the natural layout (q2 stride
N*P = 40) and the padded one (q2 stride 53, q1 stride 6, UE q2 stride N*T + 4).  The padded layout must be
conflict-free where the natural one is 2-way (stores) / 4-way (UE), without costing stage C or the point warps.
"""
import importlib.util
import pathlib

spec = importlib.util.spec_from_file_location(
    "bank", pathlib.Path(__file__).resolve().parents[1] / "tools" / "v10_stageB_bank_model.py")
bank = importlib.util.module_from_spec(spec)
spec.loader.exec_module(bank)


def test_natural_layout_stage_b_is_two_way():
    # 240 field items: warps 0-7, 24 stores each; the ideal is one wavefront per half-warp touched
    ideal_ux = bank.stageB(53, 6, 424, 1272)
    assert bank.stageB(40, 5, 320, 960) > 1.8 * ideal_ux
    assert bank.stageB(40, 5, 320, 960, False) > 1.8 * bank.stageB(53, 6, 424, 1272, False)


def test_padded_layout_keeps_stage_c_and_point_loads():
    assert bank.stageC(53, 6, 424, 1272) == bank.stageC(40, 5, 320, 960)
    assert bank.pw(53, 6) == bank.pw(40, 5) == 10   # 5 loads x 2 half-warps, conflict-free


def test_ue_padding():
    assert bank.stageBe(32) == 4 * bank.stageBe(36)
    assert bank.stageBe(36) == 16                    # 2 groups x 8 stores, one wavefront each
