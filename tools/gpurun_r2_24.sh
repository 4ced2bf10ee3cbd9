# round 2, call 24: ncu --set full of the single-pass kernel (C5, C3, C4), sanitizers over every
# kernel, C3 / C4 on the other paths (COF_SINGLE=0) for the path-choice table
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r24/san
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
COF_SINGLE=0 timeout 600 python bench.py --config C3 $B > gpurun_out/r24/C3_nosingle.jsonl 2> gpurun_out/r24/C3_nosingle.err
COF_SINGLE=0 timeout 600 python bench.py --config C4 $B > gpurun_out/r24/C4_nosingle.jsonl 2> gpurun_out/r24/C4_nosingle.err
COF_SINGLE=0 timeout 600 python bench.py --config C5 $B > gpurun_out/r24/C5_nosingle.jsonl 2> gpurun_out/r24/C5_nosingle.err
for c in C5 C3 C4; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/r24/prof_$c \
  python bench.py --config $c --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r24/prof_$c.log 2>&1
done
for t in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_cases.py > gpurun_out/r24/san/r2_$t.txt 2>&1; echo "rc=$?" >> gpurun_out/r24/san/r2_$t.txt
done
