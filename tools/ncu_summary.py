"""Summarise an ncu report for profiles/: key metrics + top source lines by stall samples.

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep > profiles/<name>.txt
"""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__grid_size",
        "launch__block_size", "launch__registers_per_thread",
        "launch__shared_mem_per_block_dynamic", "sm__inst_executed.avg.per_cycle_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_bytes.sum",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tmem_cycles_active.avg.pct_of_peak_sustained_active",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed"]


def ncu(rep, *args):
    return subprocess.run(["ncu", "-i", rep, *args], capture_output=True, text=True).stdout


def main(rep):
    raw = list(csv.reader(io.StringIO(ncu(rep, "--page", "raw", "--csv"))))
    hdr, units, vals = raw[0], raw[1], raw[2:]
    print(f"# ncu summary of {rep}")
    for v in vals:
        name = v[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
        print(f"\n## kernel: {name}")
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                print(f"{k:60s} {v[i]:>20s} {units[i]}")
        for i, h in enumerate(hdr):
            if h.startswith("smsp__average_warps_issue_stalled") and h.endswith("per_issue_active.ratio"):
                try:
                    if float(v[i]) > 0.2:
                        print(f"{h:60s} {v[i]:>20s}")
                except ValueError:
                    pass
    rows = list(csv.reader(io.StringIO(ncu(rep, "--page", "source", "--csv", "--print-source",
                                           "cuda,sass"))))
    out, hdr2, f = [], None, None
    for r in rows:
        if len(r) >= 2 and r[0] == "File Path":
            f = r[1].split("/")[-1]
            continue
        if len(r) >= 2 and r[0] == "Line No":
            hdr2 = r
            continue
        if hdr2 and len(r) > 7 and r[0]:
            try:
                out.append((float(r[4]), float(r[7]), f, r[0], r[1][:100]))
            except ValueError:
                pass
    tot = sum(o[0] for o in out) or 1
    print("\n## top source lines by warp-stall samples")
    for st, ex, f, ln, src in sorted(out, reverse=True)[:25]:
        print(f"{st / tot * 100:5.1f}%  exec {ex / 1e6:8.2f}M  {f}:{ln}  {src}")


if __name__ == "__main__":
    main(sys.argv[1])
