"""Record and summarise the per-CTA timeline of one TMA merge pass (BCF_TRACE)."""
import ctypes, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_spaa_berneys25_b200 as bcf, synthetic_inputs as si
n = 1 << 24
x = si.uniform_u32_torch(n, si.config_seed(1), torch.device("cuda:0"))
for _ in range(3):
    bcf.sort(x)
torch.cuda.synchronize()
buf = np.zeros(1 << 21, dtype=np.uint64)
bcf.lib().bcf_debug_trace_copy.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
assert bcf.lib().bcf_debug_trace_copy(buf.ctypes.data, buf.nbytes) == 0
tr = buf.reshape(-1, 256).astype(np.int64)
if os.environ.get("TRACE_SAVE"):
    np.savez_compressed(os.environ["TRACE_SAVE"], tr=tr[np.nonzero(tr[:, 0])[0]])
ctas = np.nonzero(tr[:, 0])[0]
t0 = tr[ctas, 0].min()
print("ctas", len(ctas), "kernel span us %.1f" % ((tr[ctas].max() - t0) / 1e3))
for c in list(ctas[:3]) + [ctas[len(ctas) // 2], ctas[-1]]:
    row = tr[c]
    cons = [(i, (row[1 + 4 * i] - t0) / 1e3, (row[2 + 4 * i] - t0) / 1e3, (row[3 + 4 * i] - t0) / 1e3) for i in range(16) if row[3 + 4 * i]]
    prod = [(i, (row[128 + 4 * i + 1] - t0) / 1e3 if row[128 + 4 * i + 1] else None, (row[128 + 4 * i + 2] - t0) / 1e3 if row[128 + 4 * i + 2] else None) for i in range(7) if row[128 + 4 * i + 2]]
    print("CTA", c, "start %.2f" % ((row[0] - t0) / 1e3))
    print("  consumer (tile, wait_start, data_ready, done):", [(i, round(a, 2), round(b, 2), round(d, 2)) for i, a, b, d in cons])
    print("  producer (tile, split_known, load_issued):", [(i, None if a is None else round(a, 2), round(b, 2)) for i, a, b in prod])
# aggregate: total consumer wait vs compute
waits, comps = [], []
for c in ctas:
    row = tr[c]
    for i in range(16):
        if row[3 + 4 * i]:
            waits.append(row[2 + 4 * i] - row[1 + 4 * i])
            comps.append(row[3 + 4 * i] - row[2 + 4 * i])
print("mean consumer wait per tile us %.2f, mean compute per tile us %.2f, tiles %d" % (np.mean(waits) / 1e3, np.mean(comps) / 1e3, len(waits)))
first = [tr[c][2] - tr[c][1] for c in ctas]
print("mean first-tile wait us %.2f" % (np.mean(first) / 1e3))
# detailed table for a few CTAs
for c in [ctas[0], ctas[len(ctas)//3], ctas[2*len(ctas)//3]]:
    row = tr[c]
    print("CTA", c)
    for i in range(7):
        if not row[3 + 4 * i]:
            break
        f = lambda v: "%7.2f" % ((v - t0) / 1e3) if v else "      -"
        print(f"  tile {i}: split_known {f(row[128+4*i+1])} empty_ok {f(row[128+4*i+3])} load_issued {f(row[128+4*i+2])} | wait {f(row[1+4*i])} ready {f(row[2+4*i])} done {f(row[3+4*i])}")
ends = []
starts = []
for c in ctas:
    row = tr[c]
    done = [row[3 + 4 * i] for i in range(31) if row[3 + 4 * i]]
    if done:
        ends.append((max(done) - t0) / 1e3)
    r0 = [row[2 + 4 * i] for i in range(1)]
    starts.append((row[2] - t0) / 1e3)
ends = np.array(ends)
print("CTA finish us: min %.1f p10 %.1f p50 %.1f p90 %.1f max %.1f" % tuple(np.percentile(ends, [0, 10, 50, 90, 100])))
print("first data ready us: min %.1f p50 %.1f max %.1f" % tuple(np.percentile(starts, [0, 50, 100])))
ntile = [sum(1 for i in range(31) if tr[c][3 + 4 * i]) for c in ctas]
print("tiles per CTA: min %d max %d" % (min(ntile), max(ntile)))
# per-SM view (slot 255 = smid + 1)
sm = tr[ctas, 255] - 1
if (sm >= 0).all():
    import collections
    per = collections.defaultdict(list)
    for c, s_ in zip(ctas, sm):
        row = tr[c]
        done = [row[3 + 4 * i] for i in range(31) if row[3 + 4 * i]]
        comp = [row[3 + 4 * i] - row[2 + 4 * i] for i in range(31) if row[3 + 4 * i]]
        per[int(s_)].append(((max(done) - t0) / 1e3, np.mean(comp) / 1e3, len(done)))
    fin = np.array([max(v[0] for v in per[k]) for k in sorted(per)])
    cmp_ = np.array([np.mean([v[1] for v in per[k]]) for k in sorted(per)])
    nct = np.array([len(per[k]) for k in sorted(per)])
    print("SMs", len(per), "CTAs/SM min %d max %d" % (nct.min(), nct.max()))
    print("per-SM last finish us: min %.1f p50 %.1f max %.1f" % (fin.min(), np.median(fin), fin.max()))
    print("per-SM mean tile compute us: min %.2f p50 %.2f max %.2f" % (cmp_.min(), np.median(cmp_), cmp_.max()))
    order = np.argsort(fin)
    ks = sorted(per)
    print("slowest SMs:", [(ks[i], round(fin[i], 1), round(cmp_[i], 2)) for i in order[-8:]])
    print("fastest SMs:", [(ks[i], round(fin[i], 1), round(cmp_[i], 2)) for i in order[:8]])
    # within-CTA spread of tile compute
    allc = np.array([tr[c][3 + 4 * i] - tr[c][2 + 4 * i] for c in ctas for i in range(31) if tr[c][3 + 4 * i]]) / 1e3
    print("tile compute us percentiles 10/50/90/99/max: %.2f %.2f %.2f %.2f %.2f" % tuple(np.percentile(allc, [10, 50, 90, 99, 100])))

# phase breakdown per tile: ready -> split barrier (161+3i) -> gather/merge done (160+3i) -> STS done (4+4i) -> copy-out done (3+4i)
ph = []
for c in ctas:
    row = tr[c]
    for i in range(30):
        if row[3 + 4 * i] and row[161 + 3 * i] and row[160 + 3 * i] and row[4 + 4 * i]:
            ph.append((row[161 + 3 * i] - row[2 + 4 * i], row[160 + 3 * i] - row[161 + 3 * i],
                       row[4 + 4 * i] - row[160 + 3 * i], row[3 + 4 * i] - row[4 + 4 * i]))
ph = np.array(ph) / 1e3
if len(ph):
    for k, name in enumerate(["split+origins", "lane split+gather+merge", "STS", "copy-out"]):
        print("%-24s us p10 %.2f p50 %.2f p90 %.2f mean %.2f" % ((name,) + tuple(np.percentile(ph[:, k], [10, 50, 90])) + (ph[:, k].mean(),)))
