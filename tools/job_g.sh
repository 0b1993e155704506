# ring-size / L2-persistence experiment on the C2 inspector (DRAM write-back of the boundary rings)
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for cfg in "32768 0" "2048 0" "1024 0" "32768 1" "2048 1" "1024 1"; do
  set -- $cfg
  if [ $2 = 1 ]; then export FASTZ_L2_PERSIST=1; else unset FASTZ_L2_PERSIST; fi
  FASTZ_VERBOSE=1 FASTZ_RING_ENTRIES=$1 timeout 900 ncu --metrics $M --clock-control none -k regex:k_inspect -s 1 -c 2 --csv python bench.py --profile --config 2 --no-cpu-baseline --no-secondary --no-genome-pair > gpurun_out/g_ring_$1_$2.csv 2> gpurun_out/g_ring_$1_$2.err; echo ring $1 persist $2 rc=$?
done
unset FASTZ_L2_PERSIST
for E in 32768 2048 1024; do FASTZ_RING_ENTRIES=$E timeout 600 python bench.py --steps 3 --warmup 3 --config 2 --no-cpu-baseline --no-secondary --no-genome-pair > gpurun_out/g_bench_c2_$E.json 2>&1; done
for E in 32768 2048 1024; do FASTZ_RING_ENTRIES=$E timeout 600 python bench.py --steps 3 --warmup 3 --config 3 --no-cpu-baseline --no-secondary --no-genome-pair > gpurun_out/g_bench_c3_$E.json 2>&1; done
FASTZ_L2_PERSIST=1 FASTZ_RING_ENTRIES=2048 timeout 600 python bench.py --steps 3 --warmup 3 --config 2 --no-cpu-baseline --no-secondary --no-genome-pair > gpurun_out/g_bench_c2_2048p.json 2>&1
