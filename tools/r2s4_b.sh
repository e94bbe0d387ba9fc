# A/B: K3 min-blocks 1 (current) vs 3 (<= 168 registers, 12 warps/SM) x widening from 8 / 16 / off, C2-C4.
O=gpurun_out/s4b
mkdir -p $O
L1=paper_conf_isca_libwmvgjbj025_b200/libtriosim.so
L3=paper_conf_isca_libwmvgjbj025_b200/libtriosim_mb3.so
for cfg in c2 c3 c4; do
  for lib in $L1 $L3; do
    for wf in 8 16 0; do
      for rep in 1 2; do
        TS_WIDEN_FROM=$wf TRIOSIM_LIB=$lib timeout 300 python bench.py --config $cfg --no-cpu-baseline --e2e-steps 1 2>>$O/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('$cfg', '$lib'[-12:], 'widen $wf', d['value'], d['ms_per_step'], d['roofline']['k3_ms'], d['clocks'])" >> $O/ab.txt
      done
    done
  done
done
cat $O/ab.txt
