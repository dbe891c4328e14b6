"""Summarise ncu reports: key metrics + stall reasons + SASS-region breakdown."""
import csv
import io
import subprocess
import sys

WANT = ['Kernel Name', 'gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed', 'launch__registers_per_thread', 'launch__block_size',
        'launch__grid_size', 'smsp__inst_executed.sum', 'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'launch__shared_mem_per_block_dynamic',
        'lts__t_bytes.sum']
STALLS = ['barrier', 'long_scoreboard', 'short_scoreboard', 'wait', 'lg_throttle', 'mio_throttle', 'math_pipe_throttle',
          'not_selected', 'selected', 'no_instruction', 'branch_resolving', 'dispatch_stall', 'membar', 'sleeping',
          'drain', 'imc_miss', 'tex_throttle', 'misc']


def raw(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2]


def main(rep):
    h, units, v = raw(rep)
    d = dict(zip(h, v))
    u = dict(zip(h, units))
    for w in WANT:
        if w in d:
            print(f"  {w:60s} {d[w][:80]} {u.get(w, '')}")
    tot = 0.0
    st = {}
    for s in STALLS:
        k = f'smsp__average_warps_issue_stalled_{s}_per_issue_active.ratio'
        if k in d:
            try:
                st[s] = float(d[k])
            except ValueError:
                pass
    print("  stalls (warps per issue):", ", ".join(f"{k}={v:.2f}" for k, v in sorted(st.items(), key=lambda x: -x[1]) if v > 0.05))


if __name__ == '__main__':
    for rep in sys.argv[1:]:
        print(rep)
        main(rep)
