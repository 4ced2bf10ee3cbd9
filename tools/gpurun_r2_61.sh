# round 2, call 61: e2e with a short first chunk (COF_E2E_FIRST_BASES)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r61
B="--steps 3 --warmup 3 --no-cpu --no-single-thread --no-fasta --e2e-steps 3"
for f in 0 32000000 64000000; do for c in C3 C4 C5; do
  COF_E2E_FIRST_BASES=$f timeout 600 python bench.py --config $c $B > gpurun_out/r61/${c}_$f.jsonl 2> gpurun_out/r61/${c}_$f.err; done; done
