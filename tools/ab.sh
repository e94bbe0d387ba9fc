# A/B: bench several library variants in one box (arguments: .so files)
for lib in "$@"; do
  for rep in 1 2; do
    TRIOSIM_LIB=$lib python bench.py --no-cpu-baseline --e2e-steps 1 2>>gpurun_out/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('$lib', d['value'], d['ms_per_step'], d['roofline']['k3_ms'])"
  done
done
