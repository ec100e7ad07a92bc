"""Layout check of the J/S pair swizzle of kb1_v6.cuh / kb1_v10.cuh (js_idx, restated here): every shared-memory
access pattern the C4 kernel makes on that buffer must be bank-conflict-free (ncu counted the first swizzle's
2-way conflicts; profiles/r01_kw_stage_clocks.txt).  8-byte accesses: 16 lanes of a half-warp must hit 16
distinct 8-byte banks; 16-byte accesses: 8 lanes of a quarter-warp must hit 8 distinct 16-byte slots."""

N = 8


def js_idx(col, q0):
    g = (col & 2) | ((col >> 2) & 1)
    return col * 8 + ((((q0 >> 1) ^ g) & 3) << 1) + (q0 & 1)


def test_bijective_within_row():
    for col in range(N * N):
        assert sorted(js_idx(col, q) - col * 8 for q in range(N)) == list(range(N))


def test_point_warp_accesses():
    # point warp of slab q2: lane = (q1 = lane >> 2, q0a = lane & 3); points q0a and q0a + 4
    for q2 in range(N):
        for second in (0, 4):
            for half in (0, 1):
                banks = [js_idx(q2 * N + q1, q0a + second) % 16 for q1 in range(4 * half, 4 * half + 4)
                         for q0a in range(4)]
                assert len(set(banks)) == 16


def test_dmma_fragment_accesses():
    # C^T fragments of column tile tl: lane = (lr = lane >> 2 -> row, lc = lane & 3), q0 = 4 s + lc
    for tl in range(N):
        for s in range(2):
            for half in (0, 1):
                banks = [js_idx(tl * 8 + lr, 4 * s + lc) % 16 for lr in range(4 * half, 4 * half + 4)
                         for lc in range(4)]
                assert len(set(banks)) == 16


def test_row_pair_accesses():
    # DFMA C_x stores: lanes = 8 consecutive rows, one q0 pair per instruction (16-byte slots)
    for c0 in range(0, N * N, 8):
        for pair in range(4):
            slots = [(js_idx(c, 2 * pair) % 16) // 2 for c in range(c0, c0 + 8)]
            assert len(set(slots)) == 8


def test_pct_y_slots_stay_in_the_warps_own_rows():
    """v10.wpx (PCT): point warp q2 stores Y[cd][a0][q1] at plane cd, slot q2*N^2 + a0*N + q1 (YE: j0 < 4) over J, and
    relies on every J slot of those rows belonging to its own points (lane l: q1 = l >> 2, q0 = l & 3 and l & 3 + 4),
    so no other warp's J is overwritten; the contraction warps' B^T reads the same slots."""
    for q2 in range(N):
        own = {js_idx(q2 * N + (l >> 2), (l & 3) + s) for l in range(32) for s in (0, 4)}
        assert own == set(range(q2 * N * N, (q2 + 1) * N * N))          # the warp's points fill its 64 slots
        ys = {q2 * N * N + a0 * N + q1 for a0 in range(5) for q1 in range(N)}
        assert ys <= own                                                   # Y (a0 < 5) only over its own J
        # the m8n8k4 store pattern: lane (lr = a0, lc) writes q1 = 2 lc, 2 lc + 1 -> 16-byte aligned pairs
        for lr in range(5):
            for lc in range(4):
                assert (q2 * N * N + lr * N + 2 * lc) % 2 == 0
