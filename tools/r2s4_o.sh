# widening 5-8-GPU points (TS_WIDEN_FROM=8) vs default (16) on the final kernels, C2, interleaved
O=gpurun_out/s4o
mkdir -p $O
for rep in 1 2 3; do
  for wf in 16 8; do
    TS_WIDEN_FROM=$wf timeout 300 python bench.py --config c2 --no-cpu-baseline --e2e-steps 1 2>>$O/ab.err | python -c "import json,sys; d=json.load(sys.stdin); print('c2 widen $wf', d['value'], d['ms_per_step'], d['roofline']['k3_ms'])" >> $O/ab.txt
  done
done
cat $O/ab.txt
