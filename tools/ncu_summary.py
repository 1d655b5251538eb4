"""Summarise an ncu --set full report and a launch-list CSV into profiles/.

    python tools/ncu_summary.py gpurun_out/prof_<tag>.ncu-rep gpurun_out/launches_<tag>.csv <tag>

Writes profiles/ncu_<tag>.md (per-kernel metrics + launch-list shares) and
updates profiles/ncu_traffic.json (DRAM bytes per launch, read by bench.py).
"""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def traffic_key(kernel: str, tag: str) -> str:
    """Key of a capture in profiles/ncu_traffic.json: bench.py reads the plain kernel
    name for the default (uniform, bench-configuration) capture; captures of other
    workloads keep their own key (kernel@kind)."""
    kind = next((w for w in ("biased", "single", "walk", "layer", "gather", "papers", "friendster")
                 if tag.startswith(w) or f"_{w}" in tag), None)
    return kernel.split("<")[0] + (f"@{kind}" if kind else "")
METRICS = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "lts__t_sector_hit_rate.pct": "l2_hit_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "occupancy_pct",
    "launch__registers_per_thread": "regs",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_pct",
    # sector efficiency: 32-B sectors per global-load request (1 = one sector per
    # request; 4 B useful of a 32-B sector is what a random 4-byte id costs)
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum": "ld_sectors",
    "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum": "ld_requests",
    "lts__t_sectors_srcunit_tex_op_read.sum": "l2_read_sectors",
    "lts__t_sector_op_read_hit_rate.pct": "l2_read_hit_pct",
    # NVLink (world > 1 captures)
    "nvlrx__bytes.sum": "nvl_rx",
    "nvltx__bytes.sum": "nvl_tx",
}
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "nsecond": 1e-9, "usecond": 1e-6,
              "msecond": 1e-3, "second": 1}


def raw_rows(rep):
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True,
                                  stderr=subprocess.DEVNULL)
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    return hdr, units, rows[2:]


def main(rep, launches, tag):
    hdr, units, rows = raw_rows(rep)
    stall_keys = [k for k in hdr if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")]
    kern = defaultdict(list)
    for r in rows:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        name = d["Kernel Name"].split("(")[0].replace("void ", "").strip()
        rec = {}
        for m, short in METRICS.items():
            if m in d and d[m] not in ("", "n/a"):
                v = float(d[m].replace(",", ""))
                sc = UNIT_SCALE.get(u.get(m, ""), 1)
                rec[short] = v * sc
        stalls = {}
        for k in stall_keys:
            try:
                stalls[k.replace("smsp__pcsamp_warps_issue_stalled_", "")] = float(d[k].replace(",", ""))
            except (ValueError, KeyError):
                pass
        tot = sum(stalls.values()) or 1.0
        rec["stalls"] = {k: v / tot for k, v in sorted(stalls.items(), key=lambda x: -x[1])[:5]}
        kern[name].append(rec)
    lines = [f"# ncu summary `{tag}`", "",
             f"Source: `ncu --set full --clock-control none --import-source on` (`{os.path.basename(rep)}`);"
             " cold-cache, serialised replays: absolute times are not bench values.", "",
             "| kernel | launches | duration us | DRAM read MB | DRAM write MB | DRAM % peak | L2 hit % | sectors / ld request | NVLink rx / tx MB | warps active % | regs | grid x block | top stalls |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    traffic = {}
    for name, recs in kern.items():
        n = len(recs)
        avg = lambda key: sum(r.get(key, 0.0) for r in recs) / n
        st = recs[-1]["stalls"]
        lines.append(f"| `{name}` | {n} | {avg('duration') * 1e6:.1f} | {avg('dram_read') / 1e6:.1f} | "
                     f"{avg('dram_write') / 1e6:.1f} | {avg('dram_pct'):.1f} | {avg('l2_hit_pct'):.1f} | "
                     f"{avg('ld_sectors') / max(1.0, avg('ld_requests')):.2f} | "
                     + (f"{avg('nvl_rx') / 1e6:.1f} / {avg('nvl_tx') / 1e6:.1f}" if any('nvl_rx' in r for r in recs) else "n/a")
                     + " | "
                     f"{avg('occupancy_pct'):.1f} | {int(avg('regs'))} | {int(avg('grid'))} x {int(avg('block'))} | "
                     + ", ".join(f"{k} {100 * v:.0f}%" for k, v in st.items()) + " |")
        big = max(recs, key=lambda r: r.get("dram_read", 0) + r.get("dram_write", 0))  # the fused launch
        traffic[traffic_key(name, tag)] = {"dram_bytes_per_launch": big.get("dram_read", 0) + big.get("dram_write", 0),
                         "dram_read_bytes": big.get("dram_read", 0), "dram_write_bytes": big.get("dram_write", 0),
                         "duration_s_ncu": big.get("duration", 0), "source": f"profiles/ncu_{tag}.md",
                         "note": "largest-traffic capture of this kernel (the fused sample+gather launch bench.py times)"}
    if launches and os.path.exists(launches):
        rows = list(csv.reader(open(launches)))
        start = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        h = rows[start]
        ki, vi = h.index("Kernel Name"), h.index("Metric Value")
        tot = defaultdict(float)
        cnt = defaultdict(int)
        for r in rows[start + 1:]:
            if len(r) > vi:
                nm = r[ki].split("(")[0].replace("void ", "")
                tot[nm] += float(r[vi].replace(",", ""))
                cnt[nm] += 1
        all_t = sum(tot.values())
        lines += ["", f"## Launch list (`{os.path.basename(launches)}`, `--metrics gpu__time_duration.sum`)", "",
                  "| kernel | launches | total us | mean us | share |", "|---|---|---|---|---|"]
        for nm, t in sorted(tot.items(), key=lambda x: -x[1]):
            lines.append(f"| `{nm}` | {cnt[nm]} | {t / 1e3:.1f} | {t / 1e3 / cnt[nm]:.1f} | {100 * t / all_t:.1f}% |")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", f"ncu_{tag}.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    tpath = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    old = json.load(open(tpath)) if os.path.exists(tpath) else {}
    old.update(traffic)
    json.dump(old, open(tpath, "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None, sys.argv[3] if len(sys.argv) > 3 else "r01")
