# parity tests + bench for R variants
mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
for R in ${RS:-4}; do
  FASTZ_R=$R timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_R$R.json 2> gpurun_out/bench_R$R.err
  python - <<PY
import json
d=json.loads(open("gpurun_out/bench_R$R.json").read().strip().splitlines()[-1])
print("R=$R", "GCUPS %.1f"%d["value"], "e2e %.1f"%d["e2e"]["value"], "ms %.1f"%d["ms_per_step"], "stages", {k:round(v,1) for k,v in d["stages_ms"].items()}, "roof %.3f"%d["roofline"]["frac"], "clk", d["clocks"]["sm_mhz"])
PY
done
