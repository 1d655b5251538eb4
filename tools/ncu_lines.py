"""Top CUDA source lines of an ncu --import-source capture by warp instructions
executed and stall samples: python tools/ncu_lines.py <rep> [top]"""
import csv, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout.splitlines()
rows, f, hdr = [], None, None
for r in csv.reader(out):
    if len(r) == 2 and r[0] in ("File Path", "File Name"):
        f = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = {h: i for i, h in enumerate(r)}
        continue
    if not hdr or not r or not r[0]:
        continue
    try:
        ie = int(r[hdr["Instructions Executed"]]); st = int(r[hdr["Warp Stall Sampling (All Samples)"]])
    except (ValueError, KeyError, IndexError):
        continue
    rows.append((ie, st, f, r[0], r[1][:100]))
tot = sum(x[0] for x in rows) or 1
tst = sum(x[1] for x in rows) or 1
print(f"total warp instructions {tot}, stall samples {tst}")
for x in sorted(rows, reverse=True)[:top]:
    print("%10d %5.1f%%  stall %5.1f%%  %s:%s  %s" % (x[0], 100 * x[0] / tot, 100 * x[1] / tst, x[2], x[3], x[4]))
print("-- by stall samples")
for x in sorted(rows, key=lambda x: -x[1])[:top // 2]:
    print("%10d %5.1f%%  stall %5.1f%%  %s:%s  %s" % (x[0], 100 * x[0] / tot, 100 * x[1] / tst, x[2], x[3], x[4]))
