"""Census of C3 rank-kernel rows on the host: w, a, u and the range count of the 16-tile / 4096-key range rule
for a random sample of rank rows (used to size the per-range fixed cost, profiles/r02_rank_range_cycles.txt)."""
import numpy as np, sys, time
sys.path.insert(0, '/root/repo')
import sginputs as gen
t=time.time()
H = gen.config("C3")
rp = np.asarray(H.row_ptr, dtype=np.int64); col = np.asarray(H.col, dtype=np.int64)
n = H.nrows; p = H.ncols
deg = np.diff(rp)
w = np.zeros(n, np.int64)
np.add.at(w, np.repeat(np.arange(n), deg), deg[col])
print("gen+w", time.time()-t, "W", w.sum())
thr = 870; dense = 1 << 19
rank = np.nonzero((w > thr) & (w < dense))[0]
dns = np.nonzero(w >= dense)[0]
print("rank rows", len(rank), "products", w[rank].sum(), "dense rows", len(dns), "products", w[dns].sum(), "light prod", w[w<=thr].sum())
rng = np.random.default_rng(1)
S = rng.choice(rank, 3000, replace=False)
TW=8192; RHALF=4096; RWT=16
rows=[]
for i in S:
    ks = col[rp[i]:rp[i+1]]
    cs = np.concatenate([col[rp[k]:rp[k+1]] for k in ks])
    uc = np.unique(cs)
    cnt = np.bincount(uc // TW, minlength=(p+TW-1)//TW)
    # range plan: key = (ceil(P_t/RHALF)-1, t/RWT) over tiles with cnt>0? mimic: runs of equal key, big tiles alone
    pre = np.concatenate([[0], np.cumsum(cnt)[:-1]])
    nt = len(cnt)
    key = ((pre + RHALF - 1)//RHALF - 1) * 1000 + np.arange(nt)//RWT
    big = cnt > RHALF
    st = np.ones(nt, bool)
    st[1:] = (key[1:] != key[:-1]) | big[1:] | big[:-1]
    # empty-range skipping approximated: count ranges containing >=1 entry
    rid = np.cumsum(st) - 1
    rc = np.bincount(rid, weights=cnt)
    nr = (rc > 0).sum()
    rows.append((len(ks), len(cs), len(uc), nr))
R = np.array(rows)
a, wv, u, nr = R.T
scale = w[rank].sum() / wv.sum() * len(S) / len(S)
f = len(rank)/len(S)
print("sample: a mean %.1f  w mean %.0f  u mean %.0f  ranges/row %.2f" % (a.mean(), wv.mean(), u.mean(), nr.mean()))
print("est total ranges %.3g  products/range %.0f  outputs/range %.0f" % (nr.sum()*f, wv.sum()/nr.sum(), u.sum()/nr.sum()))
for lo, hi in [(870,2048),(2048,8192),(8192,32768),(32768,131072),(131072,1<<19)]:
    m = (wv>lo)&(wv<=hi)
    print(f"w in ({lo},{hi}]: rows {m.sum()*f:.3g} prod {wv[m].sum()*f:.3g} ranges {nr[m].sum()*f:.3g} u/w {u[m].sum()/max(1,wv[m].sum()):.2f} a {a[m].mean() if m.any() else 0:.1f} u/range {u[m].sum()/max(1,nr[m].sum()):.0f}")
