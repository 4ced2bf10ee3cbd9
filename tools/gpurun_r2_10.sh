# round 2, call 10: warps per CTA x sites per lane x ring stages of the single pass, interleaved A/B
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for v in main w20r2s4 w32r1s3 w24r1s4 w28r1s4; do
  if [ $v = main ]; then L=""; else L="COF_LIB=$PWD/variants/libcof_$v.so"; fi
  for c in C5 C3 C4; do env $L timeout 600 python bench.py --config $c $B > gpurun_out/r2_b10_${v}_${c}.jsonl 2> gpurun_out/r2_b10_${v}_${c}.err; done
done
for v in w32r1s3 w28r1s4; do COF_LIB=$PWD/variants/libcof_$v.so timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -2 > gpurun_out/r2_t10_$v.log; done
timeout 600 python -m pytest tests/test_gpu_resident.py -x -q 2>&1 | tail -3 > gpurun_out/r2_t10_resident.log
