# round 2, call 15: few-blocks geometry 24/28 warps, and a spinning tile wait instead of the sleeping one
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for v in main few2426 few2424 few2824 spin spin24; do
  if [ $v = main ]; then L=""; else L="COF_LIB=$PWD/variants/libcof_$v.so"; fi
  for c in C3 C4 C2; do env $L timeout 600 python bench.py --config $c $B > gpurun_out/r2_b15_${v}_${c}.jsonl 2> gpurun_out/r2_b15_${v}_${c}.err; done
done
for v in main spin; do
  if [ $v = main ]; then L=""; else L="COF_LIB=$PWD/variants/libcof_$v.so"; fi
  env $L timeout 600 python bench.py --config C5 $B > gpurun_out/r2_b15_${v}_C5.jsonl 2> gpurun_out/r2_b15_${v}_C5.err
done
COF_LIB=$PWD/variants/libcof_few2824.so timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -2 > gpurun_out/r2_t15_few2824.log
