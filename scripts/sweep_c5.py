"""Config 5 of BASELINE.json: NTT sweep N = 2^12..2^17, L = 1..60, batch 1 and 128 ciphertexts
(2 and 256 polynomials), forward and inverse, AUTO kernel selection.  Prints one JSON line per
point: KOPS (single-prime N-point transforms per second, reading C-9) for each direction and the
HBM fraction of the algorithmic 8N bytes per transform (inputs resident; no L2 flush, so the
small points are L2-resident and latency-bound, as flagged in SURVEY.md 8.d).

usage: python scripts/sweep_c5.py [--reps 10] > gpurun_out/sweep_c5.jsonl
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=10)
    args = ap.parse_args()
    import torch
    from paper_conf_hpca_fanzzfzdtksy25_b200 import inputs, wdntt
    peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                       "MEASURED_PEAKS.json"))).get("hbm_gbs", 6550.0)
    sp = torch.cuda.current_stream().cuda_stream
    for logn in range(12, 18):
        n = 1 << logn
        for L in (1, 4, 16, 36, 60):
            primes = inputs.bench_primes(L)
            plan = wdntt.Plan(n, primes)
            for nct in (1, 128):
                b = 2 * nct
                x = inputs.uniform_residues_torch(primes, n, b, inputs.SEED_BASE + 5, device="cuda")
                y, z = torch.empty_like(x), torch.empty_like(x)
                for _ in range(2):
                    wdntt.wd_ntt_forward(plan.handle, x, y, b, sp)
                    kern = wdntt.wd_ntt_last_kernel()
                    wdntt.wd_ntt_inverse(plan.handle, y, z, b, sp)
                torch.cuda.synchronize()
                assert torch.equal(z, x), (logn, L, nct)
                # each direction's reps captured in one CUDA graph (the batch-1 points are
                # launch-bound; as bench.py --graph auto)
                cs = torch.cuda.Stream()
                cs.wait_stream(torch.cuda.current_stream())
                gf, gi = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
                with torch.cuda.graph(gf, stream=cs):
                    for _ in range(args.reps):
                        wdntt.wd_ntt_forward(plan.handle, x, y, b, cs.cuda_stream)
                with torch.cuda.graph(gi, stream=cs):
                    for _ in range(args.reps):
                        wdntt.wd_ntt_inverse(plan.handle, y, z, b, cs.cuda_stream)
                gf.replay(); gi.replay()
                torch.cuda.synchronize()
                ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
                ev[0].record()
                gf.replay()
                ev[1].record()
                gi.replay()
                ev[2].record()
                torch.cuda.synchronize()
                assert torch.equal(z, x), (logn, L, nct, "graph")
                fms = ev[0].elapsed_time(ev[1]) / args.reps
                ims = ev[1].elapsed_time(ev[2]) / args.reps
                rows = b * L
                print(json.dumps({"logN": logn, "L": L, "ciphertexts": nct, "rows": rows, "kernel": kern,
                                  "fwd_ms": fms, "inv_ms": ims,
                                  "fwd_kops": rows / fms, "inv_kops": rows / ims,
                                  "hbm_frac_fwd": rows * 8.0 * n / (fms * 1e-3) / 1e9 / peak,
                                  "bytes_in": rows * 4 * n}), flush=True)
                del x, y, z, gf, gi
            del plan
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
