"""Top source lines of an ncu report by warp-stall samples (run here, CPU).

    python tools/ncu_lines.py gpurun_out/prof.ncu-rep [N]
"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    f, hdr, agg, tot = None, None, [], 0
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            f = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr and r[0] and r[0].isdigit():
            try:
                samp = int(r[4])
                ins = int(r[7])
                thr = float(r[10]) if r[10] not in ("", "-") else 0.0
            except (ValueError, IndexError):
                continue
            tot += samp
            agg.append((samp, f, int(r[0]), ins, thr, r[1].strip()[:80]))
    agg.sort(reverse=True)
    print(f"total samples {tot}")
    for samp, f, ln, ins, thr, src in agg[:n]:
        print(f"{100.0 * samp / max(tot, 1):5.1f}% {f}:{ln:<5d} inst={ins:<10d} thr={thr:5.1f}  {src}")


if __name__ == "__main__":
    main()
