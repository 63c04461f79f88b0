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
ctas = np.nonzero(tr[:, 0])[0]
t0 = tr[ctas, 0].min()
print("ctas", len(ctas), "kernel span us %.1f" % ((tr[ctas].max() - t0) / 1e3))
for c in list(ctas[:3]) + [ctas[len(ctas) // 2], ctas[-1]]:
    row = tr[c]
    cons = [(i, (row[1 + 4 * i] - t0) / 1e3, (row[2 + 4 * i] - t0) / 1e3, (row[3 + 4 * i] - t0) / 1e3) for i in range(16) if row[3 + 4 * i]]
    prod = [(i, (row[128 + 4 * i + 1] - t0) / 1e3 if row[128 + 4 * i + 1] else None, (row[128 + 4 * i + 2] - t0) / 1e3 if row[128 + 4 * i + 2] else None) for i in range(16) if row[128 + 4 * i + 2]]
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
    for i in range(12):
        if not row[3 + 4 * i]:
            break
        f = lambda v: "%7.2f" % ((v - t0) / 1e3) if v else "      -"
        print(f"  tile {i}: split_known {f(row[128+4*i+1])} empty_ok {f(row[128+4*i+3])} load_issued {f(row[128+4*i+2])} | wait {f(row[1+4*i])} ready {f(row[2+4*i])} done {f(row[3+4*i])}")
ends = []
starts = []
for c in ctas:
    row = tr[c]
    done = [row[3 + 4 * i] for i in range(60) if row[3 + 4 * i]]
    if done:
        ends.append((max(done) - t0) / 1e3)
    r0 = [row[2 + 4 * i] for i in range(1)]
    starts.append((row[2] - t0) / 1e3)
ends = np.array(ends)
print("CTA finish us: min %.1f p10 %.1f p50 %.1f p90 %.1f max %.1f" % tuple(np.percentile(ends, [0, 10, 50, 90, 100])))
print("first data ready us: min %.1f p50 %.1f max %.1f" % tuple(np.percentile(starts, [0, 50, 100])))
ntile = [sum(1 for i in range(60) if tr[c][3 + 4 * i]) for c in ctas]
print("tiles per CTA: min %d max %d" % (min(ntile), max(ntile)))
