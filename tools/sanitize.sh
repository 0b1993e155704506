# compute-sanitizer on a small mixed workload (memcheck, racecheck, synccheck, initcheck); block-per-side forced
# (so the warp-per-side traceback runs too), plus the seeding stage on both strands and the redundant-alignment
# post-pass (K = 0, so every record is a candidate)
mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
cat > /tmp/san_case.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
from synth import genome
from paper_conf_sc_gundaboluvt21_b200 import fastz
w = genome.small_pair(90, length=8000, n_seeds=40)
with fastz.Aligner(w.T, w.Q) as a:
    r = a.extend(w.seeds)
    a.census()
    hs, an, hits = a.find_hsps(hspthresh=500)
    a.extend(an)
with fastz.Aligner(w.T, w.Q, fastz.fastz_default_params(gapped_threshold=0)) as d:
    d.extend(w.seeds)
    red, nred = d.mark_redundant()
    d.mark_redundant()
with fastz.Aligner(w.T, w.Q, fastz.fastz_default_params(options=32)) as b:
    hs2, an2, _ = b.find_hsps(pattern="1101011", hspthresh=300)
# round 2 paths: wide-ring re-inspection (forced 64-entry ring), packed contexts, LPT, predicted inspector order
os.environ["FASTZ_RING_ENTRIES"] = "64"
with fastz.Aligner(w.T, w.Q) as a:
    r2 = a.extend(w.seeds)
    a.census()
del os.environ["FASTZ_RING_ENTRIES"]
pt, pq = fastz.PackedSequence.pack(w.T), fastz.PackedSequence.pack(w.Q)
with fastz.Aligner(pt, pq) as p:
    r3 = p.extend(w.seeds)
assert r2.cigar == r.cigar and r3.cigar == r.cigar
print("ok", len(r.rec), len(hs), len(hs2), nred)
PY
for tool in memcheck racecheck synccheck initcheck; do
  FASTZ_ESCALATE_STRIPS=2 FASTZ_BLOCK_BIN=1 timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python /tmp/san_case.py > gpurun_out/san2_$tool.log 2>&1; echo "$tool rc=$?"; tail -2 gpurun_out/san2_$tool.log
done
