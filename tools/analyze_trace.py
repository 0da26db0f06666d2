"""Summarise a look-back trace written by tools/trace_lookback.py."""
import sys

import numpy as np

d = np.load(sys.argv[1])
t = d["trace"].astype(np.int64)
nb, nc, _ = t.shape
hops = (t[:, :, 2] >> 48) & 0xFF
polls = (t[:, :, 2] >> 56) & 0xFF
t &= (1 << 48) - 1
lo = t[:, :, 0][t[:, :, 0] > 0].min()
t = (t - lo) / 1000.0                          # us since first tile arrival
print(f"kernel ms {float(d['ms']):.3f}  bands {nb} chunks {nc}")
start = t[:, 0, 0]
end = t[:, -1, 3]
print("band start  (us): min %.1f med %.1f max %.1f" % (start.min(), np.median(start), start.max()))
print("band end    (us): min %.1f med %.1f max %.1f" % (end.min(), np.median(end), end.max()))
dur = end - start
print("band dur    (us): min %.1f med %.1f max %.1f" % (dur.min(), np.median(dur), dur.max()))
per = np.diff(t[:, :, 0], axis=1)
print("chunk period (us, arrival-to-arrival): med %.2f p90 %.2f" % (np.median(per), np.percentile(per, 90)))
loc = t[:, :, 1] - t[:, :, 0]
lb = t[:, :, 2] - t[:, :, 1]
st = t[:, :, 3] - t[:, :, 2]
print("arrival->local done med %.2f | local->lookback done med %.2f p90 %.2f | lookback->store med %.2f" %
      (np.median(loc), np.median(lb), np.percentile(lb, 90), np.median(st)))
lag = t[1:, :, 2] - t[:-1, :, 2]
print("inter-band lag of look-back completion (us): med %.2f p10 %.2f p90 %.2f" %
      (np.median(lag), np.percentile(lag, 10), np.percentile(lag, 90)))
ld = t[:, :, 0] - t[:, :, 4]
print("load issue->arrival med %.2f p90 %.2f" % (np.median(ld[t[:, :, 4] > -1e8]), np.percentile(ld, 90)))
print("lookback done->finish start med %.2f | finish start->stores issued med %.2f | arrival->finish start (TMEM residency) med %.2f" % (
    np.median(t[:, :, 6] - t[:, :, 2]), np.median(t[:, :, 3] - t[:, :, 6]), np.median(t[:, :, 6] - t[:, :, 0])))
b0 = t[0]
print("band0: period %.2f, load lat %.2f, arr->colr %.2f, colr->lb %.2f, lb->fin %.2f, fin->stores %.2f" % (
    np.median(np.diff(b0[:, 0])), np.median(b0[:, 0] - b0[:, 4]), np.median(b0[:, 1] - b0[:, 0]),
    np.median(b0[:, 2] - b0[:, 1]), np.median(b0[:, 6] - b0[:, 2]), np.median(b0[:, 3] - b0[:, 6])))
print("hops: mean %.2f max %d; share of chunks with hops>1: %.3f; polls mean %.2f max %d" % (hops.mean(), hops.max(), (hops > 1).mean(), polls.mean(), polls.max()))
bi = np.arange(nb)
for q in (0, 1, 2, nb // 4, nb // 2, nb - 1):
    print("  band %4d: lb med %.2f hops %.1f polls %.1f end %.1f" % (q, np.median(t[q, :, 2] - t[q, :, 1]), hops[q].mean(), polls[q].mean(), t[q, -1, 3]))
# compute-warp stall at finish(J): the add vector arrived (t6) after the
# compute warps had finished local(J + DT - 1) (t1 of that chunk)
DT = int(sys.argv[2]) if len(sys.argv) > 2 else 4
if nc > DT:
    stall = t[:, :nc - DT + 1, 6] - t[:, DT - 1:, 1]
    stall = np.maximum(stall, 0)
    print("finish stall per chunk (us): mean %.2f p50 %.2f p90 %.2f; total per band mean %.1f max %.1f" % (
        stall.mean(), np.median(stall), np.percentile(stall, 90), stall.sum(1).mean(), stall.sum(1).max()))
    for q in (0, 1, 8, nb // 4, nb // 2, 3 * nb // 4, nb - 1):
        print("  band %4d: stall total %.1f us, lb med %.2f, arrival period med %.2f" % (
            q, stall[q].sum(), np.median(t[q, :, 2] - t[q, :, 1]), np.median(np.diff(t[q, :, 0]))))
# propagation of the inclusive down the bands for a middle chunk
J = nc // 2
print("chunk %d: local done (t1) by band: " % J + " ".join("%.1f" % v for v in t[::max(1, nb // 16), J, 1]))
print("chunk %d: look-back done (t2) by band: " % J + " ".join("%.1f" % v for v in t[::max(1, nb // 16), J, 2]))
