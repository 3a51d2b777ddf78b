"""Per-source-line stall samples of one kernel in an ncu report.
python tools/src_hotspots.py rep.ncu-rep <kernel-regex> [top]"""
import csv
import io
import subprocess
import sys


def main(rep, kern, top=25):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass",
                          "--kernel-name", f"regex:{kern}"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    agg = {}
    hdr = None
    fname = "?"
    for r in rows:
        if len(r) == 2 and r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r and r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < len(hdr) or r[2] != "-":
            continue
        try:
            ln = int(r[0])
            smp = int(r[hdr.index("Warp Stall Sampling (All Samples)")])
            ins = int(r[hdr.index("Instructions Executed")])
        except ValueError:
            continue
        agg[(fname, ln)] = (smp, ins, r[1][:90])
    tot = sum(v[0] for v in agg.values()) or 1
    for (f, ln), (smp, ins, src) in sorted(agg.items(), key=lambda x: -x[1][0])[:int(top)]:
        print(f"{f[:18]:18s}:{ln:<4d} {100 * smp / tot:5.1f}%  inst={ins:>12d}  {src}")


if __name__ == "__main__":
    main(*sys.argv[1:])
