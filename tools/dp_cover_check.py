"""CPU check of the level-wise cover-existence test (reorder.cu cover_dp), same bit
loops in Python, against a brute-force exact-cover search on random compatibility
tables.  Developer tool: python tools/dp_cover_check.py"""
import itertools, random
subs=[sum(1<<i for i in c) for c in itertools.combinations(range(16),4)]
g0s=[s for s in subs if s&1]
def dp(compat):
    half=set()
    for g0 in g0s:
        if not compat[g0]: continue
        rem=~g0&0xFFFF; l1=(rem&-rem).bit_length()-1
        av=rem&~(1<<l1)
        x=av
        while x:
            bb=x&-x; y=x&(x-1)
            while y:
                cb=y&-y; z=y&(y-1)
                while z:
                    g1=(1<<l1)|bb|cb|(z&-z)
                    if compat.get(g1,0): half.add(g0|g1)
                    z&=z-1
                y&=y-1
            x&=x-1
    for u in half:
        rest=~u&0xFFFF; l2=(rest&-rest).bit_length()-1; av=rest&~(1<<l2)
        x=av
        while x:
            bb=x&-x; y=x&(x-1)
            while y:
                cb=y&-y; z=y&(y-1)
                while z:
                    g2=(1<<l2)|bb|cb|(z&-z)
                    if compat.get(g2,0) and compat.get(rest&~g2,0): return True
                    z&=z-1
                y&=y-1
            x&=x-1
    return False
def brute(compat):
    def rec(used):
        if used==0xFFFF: return True
        lo=((~used&0xFFFF)&-(~used&0xFFFF))
        for s in subs:
            if s&lo and not s&used and compat[s] and rec(used|s): return True
        return False
    return rec(0)
random.seed(1)
agree=0; pos=0
for t in range(300):
    p=random.choice([0.02,0.05,0.1,0.2])
    compat={s:(random.random()<p) for s in subs}
    a,b=dp(compat),brute(compat)
    assert a==b,(t,a,b)
    agree+=1; pos+=a
print('agree',agree,'positives',pos)
