"""Grouped-path validation sweep (run on the B200): for every matrix of the
mixed-skew suite (BASELINE.json configs[4]) and J in {32, 64, 128}, CELL at
P = 1 with Algorithm 3's widths, timed with the per-slot path (LF_GROUPED=0)
and the grouped path (LF_GROUPED=1), next to lf_cell_configure's sampled
group-union ratio and its choice (stats.spmm_grouped).  Writes OUT.jsonl and
prints a markdown table.  python scripts/grouped_sweep.py OUT.jsonl [sizes...]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402

out = sys.argv[1]
sizes = tuple(int(x) for x in sys.argv[2:]) or (1 << 18, 1 << 20)
ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731


def timed(fn, n=8):
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    a, b = ev(), ev()
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n


g = torch.Generator(device="cuda")
g.manual_seed(0)
rows = []
with open(out, "w") as f:
    for name, thunk in gen.mixed_suite(sizes, seeds=(0,)):
        A_h = thunk()
        A = lf.Csr.from_host(A_h)
        for J in (32, 64, 128):
            B = torch.rand((A_h.n_cols, J), device="cuda", generator=g) * 2 - 1
            C = torch.empty((A_h.n_rows, J), device="cuda")
            params, st = lf.configure(A, J, force_parts=1, force_format=1)
            M = lf.CellMatrix.build(A, params, st)
            rec = {"name": name, "J": J, "nnz": A_h.nnz, "e": int(params.max_width_log2[0]),
                   "ratio": st.group_union_ratio, "chosen": int(st.spmm_grouped),
                   "mean_len": st.features[3]}
            os.environ["LF_GROUPED"] = "0"
            rec["t_slot"] = timed(lambda: M.spmm(B, out=C))
            if rec["e"] <= 5:
                os.environ["LF_GROUPED"] = "1"
                rec["t_grouped"] = timed(lambda: M.spmm(B, out=C))
            os.environ.pop("LF_GROUPED", None)
            M.close()
            f.write(json.dumps(rec) + "\n")
            f.flush()
            rows.append(rec)
print("| matrix | J | e | union/nnz | mean len | chosen | per-slot ms | grouped ms | best | choice ok |")
print("|---|---|---|---|---|---|---|---|---|---|")
ok = n_el = 0
for r in rows:
    if "t_grouped" not in r:
        print(f"| {r['name']} | {r['J']} | {r['e']} | {r['ratio']:.2f} | {r['mean_len']:.1f} | - | {r['t_slot']:.3f} | - | per-slot | - |")
        continue
    best = "grouped" if r["t_grouped"] < r["t_slot"] else "per-slot"
    good = (r["chosen"] == 1) == (best == "grouped")
    n_el += 1
    ok += good
    print(f"| {r['name']} | {r['J']} | {r['e']} | {r['ratio']:.2f} | {r['mean_len']:.1f} | {r['chosen']} | "
          f"{r['t_slot']:.3f} | {r['t_grouped']:.3f} | {best} | {'yes' if good else 'NO'} |")
loss = sum(min(r["t_slot"], r["t_grouped"]) for r in rows if "t_grouped" in r)
got = sum((r["t_grouped"] if r["chosen"] else r["t_slot"]) for r in rows if "t_grouped" in r)
print(f"\nheuristic right on {ok}/{n_el} eligible cases; total time with its choices {got:.3f} ms "
      f"vs {loss:.3f} ms with the best path per case ({got / loss:.3f}x)")
