for lib in "$@"; do
  echo "== $lib"
  TRIOSIM_LIB=$lib timeout 120 python tools/latency_probe.py 16 0 1 2>&1 | grep "p="
  TRIOSIM_LIB=$lib timeout 120 python tools/latency_probe.py 16 0 1250 2>&1 | grep "p="
  TRIOSIM_LIB=$lib timeout 120 python bench.py --no-cpu-baseline --e2e-steps 1 2>>gpurun_out/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('bench', d['value'], d['ms_per_step'])"
done
