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
print("ok", len(r.rec))
PY
timeout 600 compute-sanitizer --tool memcheck --show-backtrace device python /tmp/san_case.py > gpurun_out/san_memcheck.log 2>&1; echo rc=$?
head -40 gpurun_out/san_memcheck.log
