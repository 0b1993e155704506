L=paper_conf_sc_gundaboluvt21_b200/libfastz.so
cp $L /tmp/cur.so
for rep in 1 2; do for v in n72 n80 n88; do cp ab_libs/$v.so $L; echo -n "$v "; timeout 600 python tools/n_bench.py 2>/dev/null | tail -1; done; done
cp /tmp/cur.so $L
