# round 2, call 57: masks-form search kernel timed beside the item-list one
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r57
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C4 C3 C5 C2; do timeout 300 python bench.py --config $c $B > gpurun_out/r57/$c.jsonl 2> gpurun_out/r57/$c.err; done
