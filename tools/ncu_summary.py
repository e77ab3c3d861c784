"""Key metrics of an ncu --set full report (raw page), one line per metric, for profiles/."""
import csv, subprocess, sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__grid_size", "launch__block_size",
        "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic",
        "sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_tc.avg.pct_of_peak_sustained_active",
        "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active",
        "l1tex__t_bytes.sum", "lts__t_bytes.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__cycles_active.avg.pct_of_peak_sustained_elapsed", "sm__cycles_elapsed.avg.per_second"]


def main(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        print(f"kernel: {d.get('Kernel Name', '?')[:120]}")
        for k in KEYS:
            for h, u in zip(hdr, units):
                if h == k:
                    print(f"  {k} = {d[h]} {u}")
        # tensor-pipe metrics whose exact names vary by ncu version
        for h, u in zip(hdr, units):
            if ("tensor" in h or "pipe_tc" in h or "tmem" in h) and h not in KEYS and ".avg.pct" in h \
                    and d[h] not in ("0", "") and "ops_path" not in h:
                print(f"  {h} = {d[h]} {u}")


if __name__ == "__main__":
    for rep in sys.argv[1:]:
        print(f"== {rep}")
        main(rep)
