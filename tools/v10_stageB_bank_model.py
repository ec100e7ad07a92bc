# Shared-memory bank model of kb1_v10 forward stage B stores / stage C loads (k = 4): wavefronts per zone
# for the natural U layout (q2 stride 40) and the padded PADU layouts searched over (v10.wu).
# 8-byte accesses: a warp request is two half-warps; a half-warp costs max(distinct addresses per bank).
import itertools
N,P,T=8,5,4
def wf(addrs):
    # 8-byte accesses: two half-warps, each: max multiplicity of distinct addrs per bank (addr mod 16)
    tot=0
    for h in (addrs[:16],addrs[16:]):
        d={}
        for a in set(x for x in h if x is not None):
            d.setdefault(a%16,0); d[a%16]+=1
        tot+=max(d.values()) if d else 0
    return tot
def stageB(S,R,MS,CS,ux=True):
    # items r<240 f=r//40; UX for f<3
    tot=0
    NKW=256
    for w in range(8):
        for q1 in range(8):
          for k in range(3):  # u0,u1,u2 -> m offsets 0,1,2
            addrs=[]
            for l in range(32):
                r=w*32+l
                if r<240:
                    f=r//40; r2=r%40; q2=r2//5; a0=r2%5
                    if (f<3)==ux:
                        addrs.append(f*CS + k*MS + q2*S+q1*R+a0)
                    else: addrs.append(None)
                else: addrs.append(None)
            if any(a is not None for a in addrs): tot+=wf(addrs)
    return tot
def stageC(S,R,MS,CS):
    tot=0
    for blk in range(3):
      for w in range(8):
        for a0 in range(5):
            addrs=[]
            for l in range(32):
                r=blk*256+w*32+l
                if r<576:
                    cm=r//64; col=r%64; q2=col//8; q1=col%8
                    c,m=cm//3,cm%3
                    addrs.append(c*CS+m*MS+q2*S+q1*R+a0)
                else: addrs.append(None)
            if any(a is not None for a in addrs): tot+=wf(addrs)
    return tot
# ub alone
def stageBe(SE):
    tot=0
    # e items r in 240..271 -> first 16 in blk0 (threads 240..255), 16 in blk1 threads 0..15 (non-BAL)
    for grp in (range(240,256), range(256,272)):
        for q1 in range(8):
            addrs=[]
            for r in grp:
                r2=r-240; q2=r2//4; j0=r2%4
                addrs.append(q2*SE+q1*4+j0)
            addrs += [None]*(32-len(addrs))
            tot+=wf(addrs)
    return tot
def pw(S,R):
    tot=0
    for a0 in range(5):
        addrs=[]
        for l in range(32):
            q1=(l//4)%8; addrs.append(S*0+q1*R+a0)
        tot+=wf(addrs)
    return tot


if __name__ == "__main__":
    b0=stageB(40,5,320,960); c0=stageC(40,5,320,960)
    print("current UX: B",b0,"C",c0, "ub B", stageB(40,5,320,960,False))
    res=[]
    for S in range(40,80):
      for R in range(5,10):
        if S<8*R-3: continue
        MS=8*S; MS+= (0)
        for mp in range(0,16):
          for cp in range(0,16):
            ms=MS+mp; cs=3*ms+cp
            b=stageB(S,R,ms,cs); c=stageC(S,R,ms,cs)
            res.append((b+c,b,c,S,R,mp,cp))
    res.sort(); print(res[:10])
    r2=[]
    for S in range(40,80):
      b=stageB(S,5,8*S,24*S,False); r2.append((b,S))
    r2.sort(); print("ub",r2[:5])
    print("ub S53 R6", stageB(53,6,424,3*424,False), "UX", stageB(53,6,424,1272), stageC(53,6,424,1272))
    for SE in (32,36,40,44): print("UE",SE,stageBe(SE))
    print("pw", pw(40,5), pw(53,6))

