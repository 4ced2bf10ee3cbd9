# round 2, call 21: survivor entries carried over one batch (full verification rounds), racecheck fix,
# merge_dist with a persistent shared buffer; N=2 on one GPU
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_resident.py tests/test_gpu_multi.py -x -q 2>&1 | tail -2 > gpurun_out/r2_t21.log
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C3 C4 C2 C5; do timeout 600 python bench.py --config $c $B > gpurun_out/r2_b21_${c}.jsonl 2> gpurun_out/r2_b21_${c}.err; done
timeout 1200 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_cases.py > gpurun_out/san/r2_racecheck2.txt 2>&1; echo "rc=$?" >> gpurun_out/san/r2_racecheck2.txt
COF_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29534 bench.py --gpus 2 --config C3 --steps 5 --warmup 3 > gpurun_out/r2_b21_C3_n2.jsonl 2> gpurun_out/r2_b21_C3_n2.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof21_C3 python bench.py --config C3 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
