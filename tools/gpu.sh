# One GPU session runner (run under gpurun).  Usage: MODE=<mode> TAG=<tag> bash tools/gpu.sh
#   tests   pytest -m gpu + smoke
#   bench   bench.py default line (+ reference arm)
#   launch  ncu launch list of one bench step (gpu__time_duration per launch)
#   ncu     ncu --set full of one kernel (KREGEX, default k_inspect) in one bench step
#   all     tests + bench + launch
# Output goes to gpurun_out/<tag>_*.
TAG=${TAG:-cur}
MODE=${MODE:-all}
mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null || exit 1
run_tests() {
  timeout ${TEST_TIMEOUT:-1500} python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/${TAG}_pytest.log 2>&1
  tail -3 gpurun_out/${TAG}_pytest.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; tail -2 gpurun_out/${TAG}_smoke.log
}
run_bench() {
  timeout ${BENCH_TIMEOUT:-1200} python bench.py ${BENCH_ARGS} > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
  tail -c 3000 gpurun_out/${TAG}_bench.json; tail -3 gpurun_out/${TAG}_bench.err
}
run_launch() {
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${TAG}_launches.csv \
    python bench.py --profile --no-cpu-baseline ${BENCH_ARGS} > /dev/null 2>&1; echo "launch rc=$?"
}
run_ncu() {
  timeout 1800 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-k_inspect} -s ${NCU_SKIP:-1} -c 1 \
    -o gpurun_out/${TAG}_ncu python bench.py --profile --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/${TAG}_ncu.log 2>&1; echo "ncu rc=$?"
}
case $MODE in
  tests) run_tests ;;
  bench) run_bench ;;
  launch) run_launch ;;
  ncu) run_ncu ;;
  all) run_tests; run_bench; run_launch ;;
  *) eval "$MODE" ;;
esac
ls gpurun_out | grep "^${TAG}_"
