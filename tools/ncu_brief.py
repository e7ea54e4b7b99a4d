"""One-line-per-metric summary of ncu --set full reports (duration, SM and
tensor-pipe utilisation, DRAM/L2 bytes, occupancy), for profiles/.

  python tools/ncu_brief.py gpurun_out/r5b/*.ncu-rep
"""
import csv
import subprocess
import sys

WANT = ["gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_bytes.sum", "launch__grid_size", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__cycles_active.avg"]


def main():
    for path in sys.argv[1:]:
        out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(out.splitlines()))
        if len(rows) < 3:
            print(path, "no data")
            continue
        h, u = rows[0], rows[1]
        print(f"== {path}")
        for v in rows[2:]:
            print(f"  {v[h.index('Kernel Name')]}")
            for w in WANT:
                if w in h:
                    i = h.index(w)
                    print(f"    {w:68s} {v[i]} {u[i]}")


if __name__ == "__main__":
    main()
