"""Per-step kernel shares from an ncu launch list (gpu__time_duration.sum per launch, CSV).

usage: python tools/launch_shares.py launches.csv [steps]
Census (explored-cell count) and INT32-peak launches are not part of the step and are excluded; the remaining
kernels' totals are divided by the number of fastz_extend_seeds calls in the capture (default: the number of
k_inspect launches)."""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 5]
h, data = rows[0], rows[1:]
ki, vi, mi = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Name")
tot, cnt = defaultdict(float), defaultdict(int)
for r in data:
    if r[mi] != "gpu__time_duration.sum":
        continue
    name = r[ki].split("(")[0].replace("void ", "")
    if "k_census" in name or "k_ipeak" in name:
        continue
    tot[name] += float(r[vi])
    cnt[name] += 1
steps = int(sys.argv[2]) if len(sys.argv) > 2 else max(v for k, v in cnt.items() if "k_inspect" in k)
T = sum(tot.values()) / steps
print(f"per-step kernel time {T / 1e6:.2f} ms over {steps} fastz_extend_seeds calls (cold-cache, serialised)")
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"{k[:70]:70s} {cnt[k] / steps:5.1f}/step {v / steps / 1e6:10.3f} ms {100 * v / steps / T:6.2f}%")
