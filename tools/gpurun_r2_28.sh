# round 2, call 28: one-pass look-back finder (cof_finder_scan) for the ordered item lists
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r28
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r28/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C4 C3 C5; do timeout 600 python bench.py --config $c $B > gpurun_out/r28/$c.jsonl 2> gpurun_out/r28/$c.err; done
for c in C4 C3; do COF_PATH=twocall timeout 600 python bench.py --config $c $B > gpurun_out/r28/${c}_twocall.jsonl 2> gpurun_out/r28/${c}_twocall.err; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_finder_scan -s 1 -c 1 -o gpurun_out/r28/prof_find_C4 \
  python bench.py --config C4 --steps 2 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r28/prof_find_C4.log 2>&1
