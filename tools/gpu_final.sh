# round-end capture: GPU tests, smoke, bench line, launch list, ncu full (inspector, executor), configs, seeding
TAG=${TAG:-r1e} bash tools/gpu_round.sh
for c in 1 3 5 6; do timeout 1500 python tools/config_run.py $c 16 2>&1 | tail -1 >> gpurun_out/configs_${TAG:-r1e}.jsonl; done
timeout 900 python tools/seed_bench.py 2 300000 > gpurun_out/seed_bench_${TAG:-r1e}.json 2>&1
ls gpurun_out
