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
