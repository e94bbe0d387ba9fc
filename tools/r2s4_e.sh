# list-based CTA water-filling (K3h) + head cache + cost-ordered launches: parity, phase profile, C5 subset, A/B
O=gpurun_out/s4e
mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x -k "not c5_sample" > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
TRIOSIM_LIB=paper_conf_isca_libwmvgjbj025_b200/libtriosim_prof.so timeout 600 python tools/c5_prof.py > $O/c5prof.log 2>&1
for cfg in c4 c3 c2; do
  for lib in paper_conf_isca_libwmvgjbj025_b200/libtriosim.so paper_conf_isca_libwmvgjbj025_b200/libtriosim_base.so; do
    for rep in 1 2; do
      TRIOSIM_LIB=$lib timeout 300 python bench.py --config $cfg --no-cpu-baseline --e2e-steps 1 2>>$O/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('$cfg', '$lib'[-12:], d['value'], d['ms_per_step'], d['roofline']['k3_ms'], d['clocks']['sm_mhz'], d['clocks']['samples'])" >> $O/ab.txt
    done
  done
done
timeout 1200 python tools/c5_subset.py 64 128 256 > $O/c5sub.log 2>&1; echo "rc=$?" >> $O/c5sub.log
cat $O/ab.txt
