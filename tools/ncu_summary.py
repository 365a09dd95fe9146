"""Summarise an ncu report: key SOL / memory / stall metrics per profiled launch (dev helper)."""
import csv
import io
import re
import subprocess
import sys

PAT = re.compile(r"^(gpu__time_duration.sum|dram__bytes_(read|write)\.sum|lts__t_sector_hit_rate.pct|"
                 r"syslts__t_sectors_srcunit_tex_aperture_sysmem_op_read_lookup_miss.sum|pcie__read_bytes.sum.per_second|"
                 r"sm__throughput.avg.pct_of_peak_sustained_elapsed|gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed|"
                 r"sm__warps_active.avg.pct_of_peak_sustained_active|launch__registers_per_thread|launch__grid_size|"
                 r"smsp__average_warp_latency_issue_stalled_.*|smsp__pcsamp_warps_issue_stalled_[a-z_]+$|"
                 r"dram__throughput.avg.pct_of_peak_sustained_elapsed|l1tex__t_sector_hit_rate.pct)$")


def main(path):
    raw = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"]).decode()
    rows = list(csv.reader(io.StringIO(raw)))
    h, u = rows[0], rows[1]
    for r in rows[2:]:
        print("==", r[h.index("Kernel Name")][:60], "ID", r[h.index("ID")])
        stalls = []
        for i, n in enumerate(h):
            if not PAT.match(n) or r[i] in ("", "n/a"):
                continue
            if n.startswith("smsp__pcsamp_warps_issue_stalled"):
                try:
                    stalls.append((float(r[i].replace(",", "")), n.replace("smsp__pcsamp_warps_issue_stalled_", "")))
                except ValueError:
                    pass
                continue
            print("  %-70s %s %s" % (n, r[i], u[i]))
        tot = sum(s for s, _ in stalls) or 1
        print("  stall samples:", ", ".join("%s %.0f%%" % (n, 100 * s / tot) for s, n in sorted(stalls)[::-1][:8]))


if __name__ == "__main__":
    main(sys.argv[1])
