# shared instant-time hashes in the ring fast-forward (K3, W >= 8): parity + interleaved A/B on C2 / C3
O=gpurun_out/s4n
mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
for rep in 1 2 3; do
  for cfg in c2 c3; do
    for lib in paper_conf_isca_libwmvgjbj025_b200/libtriosim.so paper_conf_isca_libwmvgjbj025_b200/libtriosim_prev.so; do
      TRIOSIM_LIB=$lib timeout 300 python bench.py --config $cfg --no-cpu-baseline --e2e-steps 1 2>>$O/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('$cfg', '$lib'[-12:], d['value'], d['ms_per_step'], d['roofline']['k3_ms'], d['clocks']['sm_mhz'])" >> $O/ab.txt
    done
  done
done
cat $O/ab.txt
