# shuffle-tree cross-warp minima (K3h CTA): parity, phase profile at 512/1024 ranks; C3 / C4 source-level K3 profile
O=gpurun_out/s4g
mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x -k "not c5_sample" > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
TRIOSIM_LIB=paper_conf_isca_libwmvgjbj025_b200/libtriosim_prof.so timeout 600 python tools/c5_prof.py 64 512 1024 > $O/c5prof.log 2>&1
for c in c3 c4; do
  timeout 900 ncu -f --set full --clock-control none --import-source on -k regex:k3_ -o /tmp/src_$c python tools/ncu_one.py $c > $O/ncu_src_$c.log 2>&1
  ncu -i /tmp/src_$c.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > $O/src_$c.csv.gz
done
ls -la $O
