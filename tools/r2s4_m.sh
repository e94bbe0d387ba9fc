# 32-bit CTA group votes: parity; wafer A/B (new vs previous build); C5 group times 64/128
O=gpurun_out/s4m
mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
for rep in 1 2; do
  for lib in paper_conf_isca_libwmvgjbj025_b200/libtriosim.so paper_conf_isca_libwmvgjbj025_b200/libtriosim_prev.so; do
    TRIOSIM_LIB=$lib timeout 400 python bench.py --config wafer --no-cpu-baseline --e2e-steps 1 2>>$O/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('wafer', '$lib'[-12:], d['value'], d['ms_per_step'], d['roofline']['k3_ms'])" >> $O/ab.txt
  done
done
timeout 600 python tools/c5_subset.py 64 128 > $O/c5sub.log 2>&1; echo "rc=$?" >> $O/c5sub.log
cat $O/ab.txt
