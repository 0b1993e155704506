# ncu full capture of the inspector for each R in $RS (reduced seed count for replay speed)
mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
for R in ${RS:-4}; do
  FASTZ_R=$R timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_inspect -c 1 -o gpurun_out/insp_R$R python bench.py --profile --no-cpu-baseline --seeds ${NSEEDS:-262144} > gpurun_out/ncu_R$R.log 2>&1
  tail -2 gpurun_out/ncu_R$R.log
done
