# round 2, call 20: sanitizers over every kernel (tools/sanitize_cases.py), 2-rank bench on one GPU,
# full bench lines with e2e / resident / FASTA
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
mkdir -p gpurun_out/san
for t in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_cases.py > gpurun_out/san/r2_$t.txt 2>&1; echo "rc=$?" >> gpurun_out/san/r2_$t.txt
done
COF_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29533 bench.py --gpus 2 --config C3 --steps 5 --warmup 3 > gpurun_out/r2_b20_C3_n2.jsonl 2> gpurun_out/r2_b20_C3_n2.err
timeout 900 python bench.py --config C5 > gpurun_out/r2_b20_C5_full.jsonl 2> gpurun_out/r2_b20_C5_full.err
for c in C3 C4 C2 C1; do timeout 900 python bench.py --config $c --no-cpu --no-single-thread > gpurun_out/r2_b20_${c}_full.jsonl 2> gpurun_out/r2_b20_${c}_full.err; done
