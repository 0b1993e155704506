MODE=tests TAG=f bash tools/gpu.sh
MODE=launch TAG=f BENCH_ARGS="--no-secondary --no-genome-pair" bash tools/gpu.sh
MODE=ncu TAG=f_exec KREGEX=k_execute BENCH_ARGS="--no-secondary --no-genome-pair" bash tools/gpu.sh
for E in 32768 4096 1024; do
  FASTZ_RING_ENTRIES=$E timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_write.sum --clock-control none -k regex:k_inspect -s 1 -c 1 --csv python bench.py --profile --config 2 --no-cpu-baseline --no-secondary --no-genome-pair > gpurun_out/f_ring_$E.csv 2>/dev/null; echo ring $E rc=$?
done
