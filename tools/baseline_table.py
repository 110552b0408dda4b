"""Render BASELINE.md §4 (round-2 results) from the committed JSON evidence in
profiles/ (bench line + tools/suite.py outputs), so the table cannot drift from
the measurements.

    python tools/baseline_table.py > /tmp/table.md
"""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
P = lambda n: json.load(open(os.path.join(ROOT, "profiles", n)))
NOM = 8000.0


def main():
    b, c3, c4 = P("r2_bench_n2.json"), P("r2_suite_c3.json"), P("r2_suite_c4.json")
    c5, n3, modes, d6 = P("r2_suite_c5.json"), P("r2_suite_n3.json"), P("r2_suite_modes.json"), P("r1_d6_cpu_oracle.json")
    peak = b["roofline"]["peak"]
    cpu = {r["workload"].split()[0]: r for r in d6["rows"]}
    rows = []
    add = rows.append
    base = b["partitions_sweep"][0]["tasks_per_s"]
    for s in b["partitions_sweep"]:
        f = s["hbm_frac"]
        add(f"| C2 GPT-2s B=1 (fill) | 1 | {s['partitions']} ({'/'.join(str(x) for x in sorted(set(s['sms']), reverse=True))}) "
            f"| {s['tasks_per_s']:.1f} | {s['tasks_per_s'] / base:.2f} | {s['p50_ms']:.0f} / {s['p99_ms']:.0f} ms | — "
            f"| {s['tasks_per_s'] * 32:.0f} | {f * peak / NOM:.2f} / {f:.2f} | C2 oracle {cpu['C2']['tasks_per_s']} tasks/s (16 cores) |")
    for s in b["partitions_sweep_equal"]:
        f = s["hbm_frac"]
        add(f"| C2 GPT-2s B=1 (equal, MIG-like) | 1 | {s['partitions']} (x{s['sms'][0]}) | {s['tasks_per_s']:.1f} "
            f"| {s['tasks_per_s'] / base:.2f} | {s['p50_ms']:.0f} / {s['p99_ms']:.0f} ms | — | {s['tasks_per_s'] * 32:.0f} "
            f"| {f * peak / NOM:.2f} / {f:.2f} | |")
    f = b["roofline"]["frac"]
    add(f"| **C2 bench step** (700 tasks/step, N2 layout {len(b['config']['partition_sms'])} x {b['config']['partition_sms'][0]} SMs) "
        f"| 1 | {len(b['config']['partition_sms'])} | **{b['value']:.1f}** | {b['value'] / base:.2f} | {b['p50_ms']:.0f} / {b['p99_ms']:.0f} ms "
        f"| {b['service_p50_ms']:.1f} / {b['service_p99_ms']:.1f} ms | {b['gen_tok_per_s']:.0f} | {f * peak / NOM:.2f} / **{f:.3f}** "
        f"| {b['cpu_baseline']['value']} tasks/s (1 task, {b['cpu_baseline']['cores']} threads) |")
    n = b["n3_shared_weights"]
    add(f"| C2 with shared weights (N3) | 1 | {len(b['config']['partition_sms'])} | {n['tasks_per_s']:.1f} | — | {n['p50_ms']:.0f} / {n['p99_ms']:.0f} ms "
        f"| — | {n['tasks_per_s'] * 32:.0f} | — / {n['hbm_frac_algorithmic']:.2f} (algorithmic bytes) | |")
    b1 = {r["batch"]: r["tasks_per_s"] for r in c3["rows"] if r["partitions"] == 1}
    for r in c3["rows"]:
        add(f"| C3 7B B={r['batch']} (14 GiB quotas) | 1 | {r['partitions']} ({'/'.join(str(x) for x in r['sms'])}) | {r['tasks_per_s']:.2f} "
            f"| {r['tasks_per_s'] / b1[r['batch']]:.2f} | {r['p50_ms']:.0f} / {r['p99_ms']:.0f} ms | {r['service_p50_ms']:.0f} / {r['service_p99_ms']:.0f} ms "
            f"| {r['gen_tok_per_s']:.0f} | {r['hbm_frac'] * peak / NOM:.2f} / {r['hbm_frac']:.2f} | 7B one layer-step {cpu['C3']['layer_step_ms']} ms (16 cores) |")
    for k in ("1", "7"):
        L = c4["layouts"][k]
        add(f"| C4 mixed decode + MPNN (1,400 tasks) | 1 | {k} | {L['tasks_per_s']:.1f} | {L['tasks_per_s'] / c4['layouts']['1']['tasks_per_s']:.2f} "
            f"| dec {L['decode']['p50_ms']:.0f} / {L['decode']['p99_ms']:.0f} ms | dec {L['decode']['service_p50_ms']:.1f}, mpnn {L['mpnn']['service_p50_ms']:.2f} ms "
            f"| — | decode {L['decode_hbm_frac']:.2f} (measured); MPNN kernel {L['mpnn_kernel_tflops']} TFLOP/s = {L['mpnn_kernel_tc_frac']:.4f} of bf16 TC peak "
            f"| MPNN oracle {cpu['C4']['tasks_per_s']} tasks/s (16 cores) |")
    pr = c5["partitioned"]["part_resize_ms"]
    for k, lab in (("partitioned", f"C5 task farm, 10k mixed, part_resize every 1,000 (p50 {pr['p50']} / p99 {pr['p99']} ms)"), ("1_partition", "C5 baseline (1,000 tasks)")):
        L = c5[k]
        add(f"| {lab} | 1 | {'7 (resized)' if k == 'partitioned' else '1'} | {L['tasks_per_s']:.1f} | {L['tasks_per_s'] / c5['1_partition']['tasks_per_s']:.2f} "
            f"| dec {L['decode']['p50_ms']:.0f} / {L['decode']['p99_ms']:.0f} ms | — | — | decode {L['decode_hbm_frac']:.2f} (measured) | |")
    print("| Config | GPUs | Partitions (SMs) | tasks/s | ratio vs N=1 | p50 / p99 completion | p50 / p99 service | gen tok/s | HBM % (nominal 8 TB/s / measured peak) | CPU oracle (cores) |")
    print("|---|---|---|---|---|---|---|---|---|---|")
    print("\n".join(rows))
    print()
    print("N1 comparison modes (`profiles/r2_suite_modes.json`, 140 GPT-2s tasks per point, tasks/s):")
    print()
    ns = sorted({r["n"] for r in modes["rows"]})
    print("| N | " + " | ".join(str(x) for x in ns) + " |")
    print("|---|" + "---|" * len(ns))
    for m in ("partitioned", "concurrent", "timeshared"):
        print(f"| {m} | " + " | ".join(f"{r['tasks_per_s']:.1f}" for n_ in ns for r in modes["rows"] if r["n"] == n_ and r["mode"] == m) + " |")
    print()
    print("N3 shared weights (`profiles/r2_suite_n3.json`, tasks/s, private vs shared, HBM held GiB):")
    print()
    print("| model | partitions | private tasks/s | shared tasks/s | private GiB | shared GiB |")
    print("|---|---|---|---|---|---|")
    keys = sorted({(r["model"], r["partitions"]) for r in n3["rows"]}, key=lambda x: (x[0], x[1]))
    for mdl, np_ in keys:
        pv = [r for r in n3["rows"] if r["model"] == mdl and r["partitions"] == np_ and r["mode"] == "private"]
        sh = [r for r in n3["rows"] if r["model"] == mdl and r["partitions"] == np_ and r["mode"] == "shared"]
        fmt = lambda L, k: (f"{L[0][k]:.2f}" if L and L[0].get(k) is not None else "—")
        print(f"| {mdl} | {np_} | {fmt(pv, 'tasks_per_s')} | {fmt(sh, 'tasks_per_s')} | {fmt(pv, 'hbm_held_gib')} | {fmt(sh, 'hbm_held_gib')} |")


if __name__ == "__main__":
    main()
