L=paper_conf_sc_gundaboluvt21_b200/libfastz.so
for v in r1d cur; do cp ab_libs/$v.so $L; echo "== $v"; timeout 300 python tools/fresh_ctx.py 2>&1 | tail -1; done
cp ab_libs/cur.so $L
CFG=2 timeout 900 python tools/ablation.py > gpurun_out/ablation_r1e.jsonl 2>&1; tail -7 gpurun_out/ablation_r1e.jsonl
