#!/usr/bin/env python
"""Summarise one round's ncu evidence into a committed text file under profiles/.

    python scripts/profile_summary.py --rep gpurun_out/TAG/prof_fused.ncu-rep \
        --launches gpurun_out/TAG/launches.csv --bench gpurun_out/TAG/bench.json \
        --det-samples 62384000 --out profiles/r01_fused_c2_summary.txt

Reads the `ncu --set full` report (raw page: time, DRAM bytes, pipe utilisation, issue
activity, stall reasons, registers, occupancy; source page: executed-instruction mix per SASS
opcode) and the `--metrics gpu__time_duration.sum` launch list (the kernel's share of the
step).  Needs the ncu CLI (present in this image; no GPU needed to read a report).
"""
import argparse
import collections
import csv
import io
import json
import subprocess

KEYS = [
    ("gpu__time_duration.sum", "duration (ns)"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("sm__cycles_elapsed.avg.per_second", "SM clock (GHz)"),
    ("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", "fp64 pipe active %"),
    ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "ALU pipe active %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe active %"),
    ("sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active", "shared pipe active %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("smsp__inst_executed.sum", "warp instructions executed"),
    ("lts__t_sectors_op_red.sum", "L2 red sectors"),
    ("lts__t_sectors_op_atom.sum", "L2 atom sectors"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate %"),
]


def ncu_csv(rep, page, extra=()):
    out = subprocess.run(["ncu", "-i", rep, "--page", page, "--csv", *extra], capture_output=True, text=True,
                         check=True).stdout
    lines = [l for l in out.splitlines() if l.startswith('"')]
    return list(csv.reader(io.StringIO("\n".join(lines))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rep", required=True)
    ap.add_argument("--launches")
    ap.add_argument("--bench")
    ap.add_argument("--det-samples", type=float, default=0.0)
    ap.add_argument("--kernel", default="pointing_to_map")
    ap.add_argument("--out", required=True)
    args = ap.parse_args()
    o = []
    raw = ncu_csv(args.rep, "raw")
    hdr, units, val = raw[0], raw[1], raw[2]
    ix = {h: i for i, h in enumerate(hdr)}
    o.append(f"# ncu --set full summary: {args.rep}")
    o.append(f"kernel: {val[ix['Kernel Name']][:160]}")
    for k, name in KEYS:
        if k in ix:
            o.append(f"{name:32s} {val[ix[k]]:>20s} {units[ix[k]]}")
    stalls = sorted(((float(val[i] or 0), h) for h, i in ix.items()
                     if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio")),
                    reverse=True)
    o.append("stall reasons (warps per issue-active cycle):")
    for v, h in stalls[:10]:
        o.append(f"  {h.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', ''):24s}"
                 f" {v:.3f}")
    if args.det_samples and "dram__bytes_read.sum" in ix:
        def to_bytes(i):
            u = units[i]
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
            return float(val[i]) * scale
        tr = to_bytes(ix["dram__bytes_read.sum"]) + to_bytes(ix["dram__bytes_write.sum"])
        o.append(f"DRAM traffic per launch {tr:.4g} B = {tr / args.det_samples:.3f} B/det-sample")
        inst = float(val[ix["smsp__inst_executed.sum"]])
        o.append(f"warp instructions per 32 det-samples {inst / (args.det_samples / 32):.1f}")
    # instruction mix from the source page
    try:
        rows = ncu_csv(args.rep, "source", ("--print-source", "sass"))
        rows = rows[next(i for i, r in enumerate(rows) if "Instructions Executed" in r):]
        h = rows[0]
        jx = {x: i for i, x in enumerate(h)}
        ops = collections.Counter()
        tot = 0
        for r in rows[1:]:
            if len(r) < len(h):
                continue
            n = int(r[jx["Instructions Executed"]] or 0)
            src = r[jx["Source"]].strip()
            op = src.split()[1] if src.startswith("@") and len(src.split()) > 1 else (src.split()[0] if src else "?")
            ops[op.split(".")[0]] += n
            tot += n
        o.append(f"executed SASS instruction mix (total {tot}):")
        for op, n in ops.most_common(24):
            per = f" = {n / (args.det_samples / 32):6.1f} per 32 det-samples" if args.det_samples else ""
            o.append(f"  {op:10s} {n:12d} {100 * n / tot:5.1f}%{per}")
    except (subprocess.CalledProcessError, KeyError) as e:
        o.append(f"(source page unavailable: {e})")
    if args.launches:
        rows = [r for r in csv.reader(open(args.launches)) if len(r) > 14 and r[12] == "gpu__time_duration.sum"]
        per = collections.defaultdict(list)
        for r in rows:
            per[r[4][:90]].append(float(r[14].replace(",", "")))
        tot = sum(sum(v) for v in per.values())
        o.append(f"launch list ({args.launches}; cold-cache, serialised — compare shares):")
        for k, v in sorted(per.items(), key=lambda kv: -sum(kv[1])):
            o.append(f"  {100 * sum(v) / tot:5.1f}%  n={len(v):3d}  mean {sum(v) / len(v) / 1e3:9.3f} us  {k}")
    if args.bench:
        for line in open(args.bench):
            if line.startswith("{"):
                b = json.loads(line)
                rf = b.get("roofline", {})
                o.append(f"bench: value {b['value']:.4g} {b['unit']}, ms/step {b['ms_per_step']:.4f}, "
                         f"kernel {rf.get('kernel_ms', 0):.4f} ms, roofline {rf.get('bound')} frac "
                         f"{rf.get('frac', 0):.3f}, clocks {b.get('clocks')}")
    open(args.out, "w").write("\n".join(o) + "\n")
    print("\n".join(o))


if __name__ == "__main__":
    main()
