# round 2, call 11: two-step survivor verification (list + cooperative verify) at w20r2s4 / w32r1s3 / w28r1s4
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for v in w20r2s4 w32r1s3 w28r1s4; do
  L="COF_LIB=$PWD/variants/libcof_$v.so"
  for c in C5 C3 C4; do env $L timeout 600 python bench.py --config $c $B > gpurun_out/r2_b11_${v}_${c}.jsonl 2> gpurun_out/r2_b11_${v}_${c}.err; done
done
COF_PATH=fused timeout 600 python bench.py --config C3 $B > gpurun_out/r2_b11_fused_C3.jsonl 2> gpurun_out/r2_b11_fused_C3.err
COF_LIB=$PWD/variants/libcof_w32r1s3.so timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -2 > gpurun_out/r2_t11_w32.log
COF_LIB=$PWD/variants/libcof_w32r1s3.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof11_w32_C5 python bench.py --config C5 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
COF_LIB=$PWD/variants/libcof_w20r2s4.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof11_w20_C3 python bench.py --config C3 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
