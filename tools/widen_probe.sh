mkdir -p gpurun_out
for L in 0 16 8; do
  TS_WIDEN_FROM=$L timeout 300 python bench.py --no-cpu-baseline --e2e-steps 2 > gpurun_out/widen_$L.json 2>&1
  python -c "
import json,sys
b=json.load(open('gpurun_out/widen_$L.json')); print('L=$L', b['value'], b['ms_per_step'], b.get('slices',{}).get('p8_per_tensor',{}).get('ms'))
"
done
for L in 0 16 8; do TS_WIDEN_FROM=$L timeout 300 python bench.py --config c3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/widen_c3_$L.json 2>&1; python -c "
import json
b=json.load(open('gpurun_out/widen_c3_$L.json')); print('c3 L=$L', b['value'], b['ms_per_step'])
"; done
TS_WIDEN_FROM=8 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/widen_pytest.log 2>&1; tail -2 gpurun_out/widen_pytest.log
