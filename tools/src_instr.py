"""Per-source-line executed instructions (warp level) of one kernel in an ncu report, sorted.
python tools/src_instr.py rep.ncu-rep <kernel-regex> [top]"""
import csv
import io
import subprocess
import sys


def main(rep, kern, top=30):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass",
                          "--kernel-name", f"regex:{kern}"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    agg, hdr, fname = {}, None, "?"
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
            ins = int(r[hdr.index("Instructions Executed")])
        except ValueError:
            continue
        if ins:
            agg[(fname, int(r[0]))] = (ins, r[1][:90])
    tot = sum(v[0] for v in agg.values()) or 1
    print(f"total {tot}")
    for (f, ln), (ins, src) in sorted(agg.items(), key=lambda x: -x[1][0])[:int(top)]:
        print(f"{f[:18]:18s}:{ln:<4d} {100 * ins / tot:5.1f}%  {ins:>12d}  {src}")


if __name__ == "__main__":
    main(*sys.argv[1:])
