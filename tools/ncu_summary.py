"""Summarise an ncu report (--set full) into profiles/: key metrics as JSON + markdown.

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep profiles/r01_tc2x512_8192 [--kernel regex]

Run here (no GPU needed): it shells out to `ncu -i ... --page raw --csv`.
"""
import csv
import io
import json
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("gpc__cycles_elapsed.max", "elapsed cycles"),
    ("gpc__cycles_elapsed.avg.per_second", "SM clock"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "tensor pipe active (of elapsed)"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor pipe active (of SM active)"),
    ("sm__ops_path_tensor_op_utchmma_src_fp16_dst_fp32_sparsity_off.sum", "UTCHMMA fp16->fp32 ops"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum", "TMA load bytes (L2->SM)"),
    ("l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum", "TMA store bytes (SM->L2)"),
    ("lts__t_sectors_srcunit_tex_op_read.sum", "L2 read sectors (from SMs)"),
    ("lts__t_sectors_srcunit_ltcfabric.sum", "L2 sectors from the die-to-die fabric"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate"),
    ("smsp__inst_executed.sum", "instructions executed"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__cluster_dim_x", "cluster x"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__shared_mem_per_block_dynamic", "dynamic smem/block"),
]


def main():
    rep, out = sys.argv[1], sys.argv[2]
    kern = None
    if "--kernel" in sys.argv:
        kern = sys.argv[sys.argv.index("--kernel") + 1]
    cmd = ["ncu", "-i", rep, "--page", "raw", "--csv"]
    if kern:
        cmd += ["-k", f"regex:{kern}"]
    txt = subprocess.run(cmd, capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = dict(zip(hdr, vals))
    u = dict(zip(hdr, units))
    summary = {"report": rep, "kernel": d.get("Kernel Name", ""), "metrics": {}}
    lines = [f"# ncu summary: `{d.get('Kernel Name', '')[:120]}`", "", f"source report: `{rep}`", "",
             "| metric | ncu name | value | unit |", "|---|---|---|---|"]
    for key, label in KEYS:
        if key in d:
            summary["metrics"][key] = {"value": d[key], "unit": u.get(key, ""), "label": label}
            lines.append(f"| {label} | `{key}` | {d[key]} | {u.get(key, '')} |")
    with open(out + ".json", "w") as f:
        json.dump(summary, f, indent=1)
    with open(out + ".md", "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
