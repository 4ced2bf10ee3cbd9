# round 2, call 14: ring depth / warps of the few-blocks geometry (C2-C4), 32 warps for C5, interleaved
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for v in main few2024 few2426 few1628; do
  if [ $v = main ]; then L=""; else L="COF_LIB=$PWD/variants/libcof_$v.so"; fi
  for c in C3 C4 C2; do env $L timeout 600 python bench.py --config $c $B > gpurun_out/r2_b14_${v}_${c}.jsonl 2> gpurun_out/r2_b14_${v}_${c}.err; done
done
for v in main many3214; do
  if [ $v = main ]; then L=""; else L="COF_LIB=$PWD/variants/libcof_$v.so"; fi
  env $L timeout 600 python bench.py --config C5 $B > gpurun_out/r2_b14_${v}_C5.jsonl 2> gpurun_out/r2_b14_${v}_C5.err
done
timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -2 > gpurun_out/r2_t14_single.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof14_C4 python bench.py --config C4 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
