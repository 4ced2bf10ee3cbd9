# round 2, call 9: v8 (uniform block offsets) at 16 / 20 / 24 warps per CTA, interleaved A/B
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for rep in 1 2; do
for v in 16 20 24; do
  if [ $v = 16 ]; then L=""; else L="COF_LIB=$PWD/variants/libcof_sw$v.so"; fi
  for c in C5 C3 C4; do env $L timeout 600 python bench.py --config $c $B > gpurun_out/r2_b9_${v}_${c}_$rep.jsonl 2> gpurun_out/r2_b9_${v}_${c}_$rep.err; done
done
done
COF_LIB=$PWD/variants/libcof_sw24.so timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -3 > gpurun_out/r2_t9w24_single.log
COF_LIB=$PWD/variants/libcof_sw20.so timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -3 > gpurun_out/r2_t9w20_single.log
