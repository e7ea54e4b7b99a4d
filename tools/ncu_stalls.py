"""Top warp-stall sites of one kernel from an ncu --set full report (source
page, SASS): the instructions with the most sampled warp stalls and their
dominant stall reasons.

  python tools/ncu_stalls.py gpurun_out/x.ncu-rep [--top 25]
"""
import argparse
import csv
import io
import subprocess


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--top", type=int, default=25)
    a = ap.parse_args()
    out = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    lines = out.splitlines()
    rows = list(csv.reader(io.StringIO("\n".join(lines[1:]))))
    h = rows[0]
    idx = {k: i for i, k in enumerate(h)}
    stall_cols = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
    data = []
    tot = 0
    for r in rows[1:]:
        try:
            n = int(r[idx["Warp Stall Sampling (All Samples)"]] or 0)
        except (ValueError, IndexError):
            continue
        tot += n
        reasons = sorted(((int(r[idx[c]] or 0), c[6:]) for c in stall_cols), reverse=True)[:3]
        data.append((n, r[idx["Address"]][-5:], r[idx["Source"]].strip()[:70], reasons))
    data.sort(reverse=True)
    print(f"{lines[0][:120]}\ntotal samples {tot}")
    for n, ad, src, rs in data[:a.top]:
        print(f"{100 * n / max(1, tot):5.1f}% {ad} {src:70s} {' '.join(f'{c}:{k}' for k, c in rs if k)}")


if __name__ == "__main__":
    main()
