"""One-screen summary of an ncu --set full capture (run here, on the CPU box):

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep [label] >> profiles/ncu_r2_single.md

Duration, issue-slot use, pipe utilisation, warp-stall reasons, DRAM traffic per launch,
executed instructions, and the hottest 80-instruction SASS regions by executed
instructions and stall samples (the map from regions to source is in DESIGN.md §5)."""
import collections
import csv
import subprocess
import sys


def raw_metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    return rows[0], rows[1], rows[2:]


def main():
    rep = sys.argv[1]
    label = sys.argv[2] if len(sys.argv) > 2 else rep
    hdr, units, rows = raw_metrics(rep)
    print(f"### {label}\n")
    want = {
        "gpu__time_duration.sum": "duration",
        "sm__inst_executed.sum": "executed warp instructions",
        "sm__issue_active.avg.pct_of_peak_sustained_active": "issue slots busy %",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active": "ALU pipe %",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active": "FMA pipe %",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active": "LSU pipe %",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active": "XU pipe %",
        "smsp__warps_eligible.avg.per_cycle_active": "eligible warps / scheduler",
        "dram__bytes_read.sum": "DRAM bytes read",
        "dram__bytes_write.sum": "DRAM bytes written",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed": "DRAM throughput %",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum": "shared bank conflicts",
        "launch__registers_per_thread": "registers / thread",
        "launch__block_size": "block size",
        "launch__grid_size": "grid size",
    }
    for r in rows[:1]:
        name = r[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
        print(f"kernel: `{name[:140]}`\n")
        print("| metric | value |\n|---|---|")
        for k, lab in want.items():
            if k in hdr:
                i = hdr.index(k)
                print(f"| {lab} | {r[i]} {units[i]} |")
        stalls = []
        for i, n in enumerate(hdr):
            if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio"):
                try:
                    v = float(r[i])
                except ValueError:
                    continue
                if v >= 0.1:
                    stalls.append((v, n[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
        print("\nwarp stalls per issued instruction: " + ", ".join(f"{n} {v:.2f}" for v, n in sorted(stalls, reverse=True)))
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    srows = list(csv.reader(out.splitlines()))
    if len(srows) > 2:
        h = srows[1]
        iI, iS = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
        seq = []
        for r in srows[2:]:
            src = r[1].strip()
            op = (src.split()[1] if src.startswith("@") else src.split()[0]).split(".")[0] if src else ""
            seq.append((op, int(r[iI] or 0), int(r[iS] or 0)))
        tot = sum(x[1] for x in seq) or 1
        tots = sum(x[2] for x in seq) or 1
        print("\n| SASS region | instructions | stall samples | top opcodes |\n|---|---|---|---|")
        for b in range(0, len(seq), 80):
            blk = seq[b:b + 80]
            n = sum(x[1] for x in blk)
            st = sum(x[2] for x in blk)
            if n / tot > 0.02 or st / tots > 0.02:
                ops = collections.Counter(x[0] for x in blk if x[1] > 0)
                print(f"| {b}-{b + 79} | {n / tot * 100:.1f} % | {st / tots * 100:.1f} % | "
                      + ", ".join(f"{k} {v}" for k, v in ops.most_common(5)) + " |")
    print()


if __name__ == "__main__":
    main()
