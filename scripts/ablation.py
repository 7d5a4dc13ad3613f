"""The paper's version ablation (Fig.12-13: Pruning, Reorder on top of the baseline),
re-done on one B200 for every synthetic family, plus the B200-specific fusion ablation.

For each family at n qubits, circuit seconds (device CUDA events around qgpu_state_reset +
qgpu_apply_circuit on the state's stream, median of --reps after one warm-up) for:
  base      prune=0 reorder=0   every pass over the full 2^n state, program order
  prune     prune=1 reorder=0   Alg.1 pruning / delayed involvement, program order
  greedy    prune=1 reorder=1   + Alg.2 greedy reorder
  forward   prune=1 reorder=2   + Alg.3 forward-looking reorder (the default)
  unfused   prune=1 reorder=2 fuse_bits=0   one gate per HBM pass (the paper's granularity)
with the pruning statistics (live amplitudes processed / full, Table II "ops before full
involvement"). Writes one JSON object per family to --out (JSON lines) and prints a table.

    python scripts/ablation.py [--n 30] [--families qft,qaoa,gs,hlf,iqp,bv,rqc] [--out f.jsonl]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

VERSIONS = [("base", dict(prune=0, reorder=0)), ("prune", dict(prune=1, reorder=0)),
            ("greedy", dict(prune=1, reorder=1)), ("forward", dict(prune=1, reorder=2)),
            ("unfused", dict(prune=1, reorder=2, fuse_bits=0))]
REFINED = ("refined", dict(prune=1, reorder=2, involve_rule=1))  # NEXT-1 (--refined)

# --host-slice-bits h: the paper's own setting (state in host memory) on the host tier
# (NEXT-2). The paper applies one gate per traversal of the chunks, so its versions are unfused:
#   base_u    prune=0 reorder=0 fuse_bits=0   every gate streams the whole state (Baseline+Overlap)
#   prune_u   prune=1 reorder=0 fuse_bits=0   + pruning / delayed involvement (Pruning)
#   forward_u prune=1 reorder=2 fuse_bits=0   + Alg.3 reorder (Reorder)
#   forward   prune=1 reorder=2               + B200 fusion: one sweep per run of passes
#   compressed                                + GFC on the host link (the paper's Compression)
# paper_*: one sweep of the slices per gate (QGPU_HOST_SWEEP_PER_PASS=1), the paper's traversal
HOST_VERSIONS = [("paper_base", dict(prune=0, reorder=0, fuse_bits=0, per_pass=1)),
                 ("paper_prune", dict(prune=1, reorder=0, fuse_bits=0, per_pass=1)),
                 ("paper_reorder", dict(prune=1, reorder=2, fuse_bits=0, per_pass=1)),
                 ("base_u", dict(prune=0, reorder=0, fuse_bits=0)),
                 ("prune_u", dict(prune=1, reorder=0, fuse_bits=0)),
                 ("forward_u", dict(prune=1, reorder=2, fuse_bits=0)),
                 ("forward", dict(prune=1, reorder=2)),
                 ("refined", dict(prune=1, reorder=2, involve_rule=1)),
                 ("compressed", dict(prune=1, reorder=2, host_compress=1))]  # + GFC on the link


def family(name, n):
    from workloads import circuits as wc
    if name == "qft":
        return wc.qft(n)
    if name == "qaoa":
        return wc.qaoa(n, 2, seed=1)
    if name == "rqc":
        return wc.rqc(n, 20, seed=3)
    if name in ("gs", "hlf"):
        r = 1
        for k in range(1, int(n ** 0.5) + 1):
            if n % k == 0:
                r = k
        return wc.gs(r, n // r) if name == "gs" else wc.hlf(r, n // r, seed=2)
    if name == "iqp":
        return wc.iqp(n)
    if name == "bv":
        return wc.bv(n, (0b1011 * 0x11111111) & ((1 << (n - 1)) - 1))
    raise SystemExit(f"unknown family {name}")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=30)
    ap.add_argument("--families", default="qft,qaoa,gs,hlf,iqp,bv,rqc")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--unfused-max-gates", type=int, default=1200)
    ap.add_argument("--out", default=None)
    ap.add_argument("--host-slice-bits", type=int, default=0)
    ap.add_argument("--paper-max-gates", type=int, default=500,
                    help="host tier: skip the one-sweep-per-gate versions above this many gates")
    ap.add_argument("--refined", action="store_true", help="also the refined involvement rule (NEXT-1)")
    args = ap.parse_args()
    global VERSIONS
    host = args.host_slice_bits
    if host:
        VERSIONS = HOST_VERSIONS
    elif args.refined:
        VERSIONS = VERSIONS + [REFINED]
    import torch
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q
    q.load()
    stream = torch.cuda.Stream()
    rows = []
    for fam in args.families.split(","):
        c = family(fam, args.n)
        circ = q.Circuit(c.qasm())
        ngates = circ.info()[1]
        res = {"family": fam, "n": args.n, "gates": ngates, "host_slice_bits": host}
        for vname, cfg in VERSIONS:
            if vname.startswith("unfused") and ngates > args.unfused_max_gates:
                continue
            cfg = dict(cfg)
            os.environ["QGPU_HOST_SWEEP_PER_PASS"] = str(cfg.pop("per_pass", 0))
            if cfg.get("per_pass_skip") or (host and "paper" in vname and ngates > args.paper_max_gates):
                continue
            st = q.State(args.n, stream=stream.cuda_stream, host_slice_bits=host, timing=1 if host else 0, **cfg)
            times = []
            for it in range(1 + args.reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                st.reset()
                st.apply_circuit(circ)
                e1.record(stream)
                e1.synchronize()
                if it:
                    times.append(e0.elapsed_time(e1))
            s = st.stats()
            st.close()
            res[vname] = {"ms": statistics.median(times), "passes": s["passes"],
                          "live_frac": s["amps_processed"] / max(s["amps_full"], 1),
                          "ops_before_full_involvement": s["ops_before_full_involvement"]}
            if host:
                res[vname].update(sweeps=s["host_runs"], slice_loads=s["host_slice_loads"],
                                  slice_skips=s["host_slice_skips"],
                                  link_GB=(s["host_h2d_bytes"] + s["host_d2h_bytes"]) / 1e9)
        rows.append(res)
        print(json.dumps(res), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")
    if host:
        print(f"\nhost tier 2^{host} slices, n={args.n}: circuit ms (link GB, sweeps)")
        for r in rows:
            print(f"{r['family']:8} {r['gates']:6d} " + " ".join(
                f"{v}={r[v]['ms']:.0f}ms({r[v]['link_GB']:.0f}GB,{r[v]['sweeps']})" for v, _ in VERSIONS if v in r))
        return
    print(f"\n{'family':8} {'gates':>6} " + " ".join(f"{v:>10}" for v, _ in VERSIONS) +
          "   prune/base forward/prune live%(fwd) TableII(prog->fwd)")
    for r in rows:
        ms = [r[v]["ms"] if v in r else float("nan") for v, _ in VERSIONS]
        print(f"{r['family']:8} {r['gates']:6d} " + " ".join(f"{m:10.3f}" for m in ms) +
              f"   {ms[1] / ms[0]:10.3f} {ms[3] / ms[1]:12.3f} {100 * r['forward']['live_frac']:9.1f}"
              f"   {r['prune']['ops_before_full_involvement']}->{r['forward']['ops_before_full_involvement']}")


if __name__ == "__main__":
    main()
