# K3 CTAs of 64 threads (2 warps: 5 CTAs / 10 warps per SM at ~190 registers) vs 128 (2 CTAs / 8 warps), C2-C4
O=gpurun_out/s4p
mkdir -p $O
for rep in 1 2; do
  for cfg in c2 c3 c4; do
    for lib in paper_conf_isca_libwmvgjbj025_b200/libtriosim.so paper_conf_isca_libwmvgjbj025_b200/libtriosim_t64.so; do
      TRIOSIM_LIB=$lib timeout 300 python bench.py --config $cfg --no-cpu-baseline --e2e-steps 1 2>>$O/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('$cfg', '$lib'[-12:], d['value'], d['ms_per_step'], d['roofline']['k3_ms'])" >> $O/ab.txt
    done
  done
done
cat $O/ab.txt
