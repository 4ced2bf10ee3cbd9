# round 2, call 41: FASTA end to end (cli.run) after sizing search_host's buffers from the first chunk
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r41
timeout 600 python -m pytest tests/test_cli.py tests/test_gpu_resident.py -x -q > gpurun_out/r41/tests.log 2>&1
for c in C5 C4 C3; do timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --no-single-thread > gpurun_out/r41/$c.jsonl 2> gpurun_out/r41/$c.err; done
