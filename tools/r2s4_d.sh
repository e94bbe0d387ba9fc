# warp-0 progressive filling for CTA points (K3h) + head-operator cache (K3 PIPE / K3h): parity, phase profile,
# A/B on C2-C4, C5 subset K3 times per N
O=gpurun_out/s4d
mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x -k "not c5_sample" > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
TRIOSIM_LIB=paper_conf_isca_libwmvgjbj025_b200/libtriosim_prof.so timeout 600 python tools/c5_prof.py > $O/c5prof.log 2>&1
for cfg in c4 c3 c2; do
  for lib in paper_conf_isca_libwmvgjbj025_b200/libtriosim.so paper_conf_isca_libwmvgjbj025_b200/libtriosim_wf.so; do
    for rep in 1 2; do
      TRIOSIM_LIB=$lib timeout 300 python bench.py --config $cfg --no-cpu-baseline --e2e-steps 1 2>>$O/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('$cfg', '$lib'[-12:], d['value'], d['ms_per_step'], d['roofline']['k3_ms'], d['clocks']['sm_mhz'], d['clocks']['samples'])" >> $O/ab.txt
    done
  done
done
timeout 900 python tools/c5_subset.py 64 128 256 > $O/c5sub.log 2>&1; echo "rc=$?" >> $O/c5sub.log
cat $O/ab.txt
