# round 2, call 17: chunk grabbing from the CTA ring (no fixed word ownership)
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_resident.py -x -q 2>&1 | tail -2 > gpurun_out/r2_t17_single.log
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for v in main few2424 few2824; do
  if [ $v = main ]; then L=""; else L="COF_LIB=$PWD/variants/libcof_$v.so"; fi
  for c in C3 C4 C2; do env $L timeout 600 python bench.py --config $c $B > gpurun_out/r2_b17_${v}_${c}.jsonl 2> gpurun_out/r2_b17_${v}_${c}.err; done
done
for v in main many3213; do
  if [ $v = main ]; then L=""; else L="COF_LIB=$PWD/variants/libcof_$v.so"; fi
  env $L timeout 600 python bench.py --config C5 $B > gpurun_out/r2_b17_${v}_C5.jsonl 2> gpurun_out/r2_b17_${v}_C5.err
done
COF_LIB=$PWD/variants/libcof_few2424.so timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -2 > gpurun_out/r2_t17_few2424.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof17_C4 python bench.py --config C4 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof17_C3 python bench.py --config C3 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
