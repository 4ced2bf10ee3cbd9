# round 2, call 36: e2e pipeline traces (COF_TRACE) of C3 with and without the split fill
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r36
B="--steps 3 --warmup 3 --no-cpu --no-single-thread --no-fasta --e2e-steps 2"
COF_TRACE=1 timeout 600 python bench.py --config C3 $B > gpurun_out/r36/C3_trace.jsonl 2> gpurun_out/r36/C3_trace.err
COF_TRACE=1 COF_SPLIT_FILL=1 timeout 600 python bench.py --config C3 $B > gpurun_out/r36/C3_trace_split.jsonl 2> gpurun_out/r36/C3_trace_split.err
COF_TRACE=1 timeout 600 python bench.py --config C5 $B > gpurun_out/r36/C5_trace.jsonl 2> gpurun_out/r36/C5_trace.err
