import numpy as np
rng=np.random.default_rng(1)
# C4-like block segment: rows with power-law lengths, block share 1/4, random columns in 25K
def seg_rows(n_entries):
    rows=[]
    tot=0
    while tot<n_entries:
        u=rng.random(); L=min(100000,int(13.64*(1-u)**(-1/1.5)))
        Lb=rng.binomial(L,0.25)
        if Lb==0: continue
        rows.append(Lb); tot+=Lb
    return rows
def window_stats(cols, rids, greedy):
    # cols: 256 entries (lane l: 8l..8l+7)
    c=cols.reshape(32,8).copy(); r=rids.reshape(32,8)
    if greedy:
        for e in range(8):
            cnt=np.zeros(32,int)
            for l in range(32):
                # candidates: positions j>=e in lane l with r[l,j]==r[l,e]
                cand=[j for j in range(e,8) if r[l,j]==r[l,e]]
                best=min(cand,key=lambda j:cnt[c[l,j]%32])
                c[l,e],c[l,best]=c[l,best],c[l,e]
                cnt[c[l,e]%32]+=1
    loads=[np.bincount(c[:,e]%32,minlength=32).max() for e in range(8)]
    return np.mean(loads)
base=[];gr=[]
for w in range(300):
    rows=seg_rows(256)
    rid=np.concatenate([np.full(L,i) for i,L in enumerate(rows)])[:256]
    cols=rng.integers(0,25000,256)
    base.append(window_stats(cols,rid,False)); gr.append(window_stats(cols,rid,True))
print("mean max-bank-load per slot: random %.2f greedy %.2f"%(np.mean(base),np.mean(gr)))
def window_stats2(cols, rids, passes=3):
    c=cols.reshape(32,8).copy(); r=rids.reshape(32,8)
    for e in range(8):
        cnt=np.zeros(32,int)
        cands={l:[j for j in range(e,8) if r[l,j]==r[l,e]] for l in range(32)}
        order=sorted(range(32),key=lambda l:len(cands[l]))
        for l in order:
            best=min(cands[l],key=lambda j:cnt[c[l,j]%32])
            c[l,e],c[l,best]=c[l,best],c[l,e]
            cnt[c[l,e]%32]+=1
    loads=[np.bincount(c[:,e]%32,minlength=32).max() for e in range(8)]
    return np.mean(loads)
g2=[]
rng=np.random.default_rng(1)
for w in range(300):
    rows=seg_rows(256)
    rid=np.concatenate([np.full(L,i) for i,L in enumerate(rows)])[:256]
    cols=rng.integers(0,25000,256)
    g2.append(window_stats2(cols,rid))
print("ordered greedy %.2f"%np.mean(g2))

def greedy2(c,r):  # the ordered greedy of k_pk_bankopt (fewest-choice lanes first)
    c=c.copy()
    for e in range(8):
        cnt=np.zeros(32,int)
        cands={l:[j for j in range(e,8) if r[l,j]==r[l,e]] for l in range(32)}
        for l in sorted(range(32),key=lambda l:len(cands[l])):
            best=min(cands[l],key=lambda j:cnt[c[l,j]%32])
            c[l,e],c[l,best]=c[l,best],c[l,e]
            cnt[c[l,e]%32]+=1
    return c
# + the local search of k_pk_bankopt (round 2c): slot-to-slot swaps inside a lane
def loads(c):
    return np.array([np.bincount(c[:,e]%32,minlength=32) for e in range(8)])  # [slot][bank]
def local_search(c,r,iters=200):
    c=c.copy()
    L=loads(c)
    for it in range(iters):
        improved=False
        # cost = sum over slots of max load (what the hardware pays)
        for e in range(8):
            m=L[e].max()
            if m<=1: continue
            banks=np.where(L[e]==m)[0]
            for b in banks:
                lanes=[l for l in range(32) if c[l,e]%32==b]
                done=False
                for l in lanes:
                    for f in range(8):
                        if f==e or r[l,f]!=r[l,e]: continue
                        b2=c[l,f]%32
                        if b2==b: continue
                        # swap entries between slots e,f in lane l
                        # new loads: slot e: b-1, b2+1 ; slot f: b2-1, b+1
                        if L[e][b2]+1 < m and L[f][b]+1 <= L[f].max() and L[f][b]+1 < m+0:
                            L[e][b]-=1;L[e][b2]+=1;L[f][b2]-=1;L[f][b]+=1
                            c[l,e],c[l,f]=c[l,f],c[l,e]
                            done=True;improved=True;break
                    if done: break
        if not improved: break
    return c
def lb(c,r):
    # per slot bound: a bank with degree d over the 8 slots forces max load >= ceil(d/8) somewhere
    deg=np.bincount((c%32).ravel(),minlength=32)
    return deg.max()/8
res={'rand':[], 'greedy':[], 'ls':[], 'bound':[]}
rng=np.random.default_rng(1)
for w in range(300):
    rows=seg_rows(256)
    rid=np.concatenate([np.full(L,i) for i,L in enumerate(rows)])[:256].reshape(32,8)
    cols=rng.integers(0,25000,256).reshape(32,8)
    res['rand'].append(loads(cols).max(1).mean())
    g=greedy2(cols,rid); res['greedy'].append(loads(g).max(1).mean())
    s=local_search(g,rid); res['ls'].append(loads(s).max(1).mean())
    res['bound'].append(lb(cols,rid))
print({k:round(float(np.mean(v)),3) for k,v in res.items()})
