"""Per-source-line instruction counts and stall samples of one kernel from an ncu report.

    python tools/ncu_lines.py <report.ncu-rep> <kernel regex> [top]
"""
import csv
import subprocess
import sys


def main():
    rep, kern = sys.argv[1], sys.argv[2]
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "--kernel-name", f"regex:{kern}"], capture_output=True, text=True).stdout
    cur, agg = None, []
    for r in csv.reader(src.splitlines()):
        if len(r) >= 2 and r[0] == "File Path":
            cur = r[1].split("/")[-1]
            continue
        if cur and len(r) > 8 and r[0].isdigit():
            try:
                ie, st = int(r[7] or 0), int(r[4] or 0)
            except ValueError:
                continue
            if ie or st:
                agg.append((ie, st, cur, int(r[0]), r[1].strip()[:100]))
    tot = sum(a[0] for a in agg) or 1
    tst = sum(a[1] for a in agg) or 1
    print(f"warp instructions {tot}, stall samples {tst}")
    for ie, st, f, l, t in sorted(agg, reverse=True)[:top]:
        print(f"{100 * ie / tot:5.1f}% inst {100 * st / tst:5.1f}% stall  {f}:{l}  {t}")


if __name__ == "__main__":
    main()
