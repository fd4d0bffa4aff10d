"""Markdown status table from a bench.py JSON line (the headline plus `configs`): workload, kernel,
GCUPS, ms, binding roofline term and its fraction, parity.  Used for README / DESIGN / BASELINE.

    python tools/status_table.py profiles/round2_bench.json
"""
import json
import sys


def main():
    line = [l for l in open(sys.argv[1]) if l.strip().startswith("{")][-1]
    d = json.loads(line)
    rows = [(d["config"]["workload"], d)] + list((d.get("configs") or {}).items())
    print("| config | kernel | GCUPS | ms / fill | binding term | frac | parity |")
    print("|---|---|---|---|---|---|---|")
    for name, r in rows:
        rf = r.get("roofline", {})
        plan = r.get("plan", {})
        par = r.get("parity", {})
        print(f"| {name} | {plan.get('kernel', '?')} | {r['value']:.1f} | {r['ms_per_step']:.4f} | "
              f"{rf.get('bound', '?')} | {rf.get('frac', 0):.3f} | {'match' if par.get('match') else par} |")
    if d.get("e2e"):
        print(f"\ne2e ({d['config']['workload']}, host buffers through lddp_fill_host): {d['e2e']['value']} {d['e2e']['unit']}")
    if d.get("cpu_baseline"):
        c = d["cpu_baseline"]
        print(f"cpu_baseline: {c.get('value')} {c.get('unit')} on {c.get('cores')} core(s), {c.get('sample')}")


if __name__ == "__main__":
    main()
