# round 2, call 50: resident-genome chunk size (the records' D2H tail after the last chunk)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r50
B="--steps 3 --warmup 3 --no-cpu --no-single-thread --no-fasta --e2e-steps 3"
for r in 800000000 400000000 200000000; do for c in C5 C3; do
  COF_RESIDENT_CHUNK_BASES=$r timeout 600 python bench.py --config $c $B > gpurun_out/r50/${c}_$r.jsonl 2> gpurun_out/r50/${c}_$r.err; done; done
