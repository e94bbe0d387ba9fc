# A/B: bench several library variants in one box.  Usage: bash tools/ab.sh "c2 c3 c4" lib1.so lib2.so ...
cfgs="$1"; shift
for cfg in $cfgs; do
  for lib in "$@"; do
    for rep in 1 2; do
      TRIOSIM_LIB=$lib timeout 300 python bench.py --config $cfg --no-cpu-baseline --e2e-steps 1 2>>gpurun_out/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('$cfg', '$lib', d['value'], d['ms_per_step'], d['roofline']['k3_ms'])"
    done
  done
done
