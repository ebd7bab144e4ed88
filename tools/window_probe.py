"""Window-protocol proxy on one GPU (diagnostic): the configs[1] and COMB
exchanges with every self message forced through the multi-GPU window path
(DDT_SELF_VIA_WINDOW=1: pack -> window -> flag / LL -> unpack, one exchange
kernel) vs the default DirectIPC step, timed exactly like bench.py (K-step
CUDA graph over R rotating replicas, L2 read sweep before the timed replay).
Variants are built first (knobs are read at plan creation), then timed
round-robin; medians over rounds.  Usage: python tools/window_probe.py [cfg1|comb|all]"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import FACE_DIRS, ALL_DIRS  # noqa: E402

VARIANTS = {
    "direct": {},
    "direct_nopair": {"DDT_NO_PAIR": "1"},
    "direct_grid0": {"DDT_GRID_MODE": "0"},
    "direct_grid1": {"DDT_GRID_MODE": "1"},
    "direct_nospread": {"DDT_SPREAD": "0"},
    "direct_ub2": {"DDT_SPREAD_UB": "2"},
    "direct_dense4": {"DDT_SPREAD_DENSE_UB": "4"},
    "direct_dense2": {"DDT_SPREAD_DENSE_UB": "2"},
    "window": {"DDT_SELF_VIA_WINDOW": "1"},
    "pdirect": {"DDT_SELF_VIA_DIRECT": "1", "_mode": "p2p_direct"},
    "pdirect_sys": {"DDT_SELF_VIA_DIRECT": "1", "DDT_FORCE_SYS_SCOPE": "1", "_mode": "p2p_direct"},
    "window_sys": {"DDT_SELF_VIA_WINDOW": "1", "DDT_FORCE_SYS_SCOPE": "1"},
    "window_xgrid1": {"DDT_SELF_VIA_WINDOW": "1", "DDT_XGRID_MODE": "1"},
    "window_xgrid2": {"DDT_SELF_VIA_WINDOW": "1", "DDT_XGRID_MODE": "2"},
    "window_claim1": {"DDT_SELF_VIA_WINDOW": "1", "DDT_XGRID_MODE": "1", "DDT_XCLAIM": "1"},
    "window_claim16": {"DDT_SELF_VIA_WINDOW": "1", "DDT_XGRID_MODE": "1", "DDT_XCLAIM": "16"},
    "window_noll": {"DDT_SELF_VIA_WINDOW": "1", "DDT_NO_LL": "1"},
    "window_g2": {"DDT_SELF_VIA_WINDOW": "1", "DDT_XONCE_G": "2"},
    "window_xub2": {"DDT_SELF_VIA_WINDOW": "1", "DDT_XUB_SMALL": "2"},
    "window_g4": {"DDT_SELF_VIA_WINDOW": "1", "DDT_XONCE_G": "4"},
    "window_noxpair": {"DDT_SELF_VIA_WINDOW": "1", "DDT_NO_XPAIR": "1"},
    "window_llub2": {"DDT_SELF_VIA_WINDOW": "1", "DDT_XUB_LL": "2"},
    "window_llub2_x1": {"DDT_SELF_VIA_WINDOW": "1", "DDT_XUB_LL": "2", "DDT_XGRID_MODE": "1", "DDT_XCLAIM": "1"},
}


def build(cfg, names):
    wls = {}
    base_env = dict(os.environ)
    for n in names:
        for k in ("DDT_SELF_VIA_WINDOW", "DDT_XGRID_MODE", "DDT_XCLAIM", "DDT_NO_LL", "DDT_NO_PAIR", "DDT_SPREAD_UB", "DDT_SPREAD_DENSE_UB", "DDT_XUB_LL", "DDT_NO_XPAIR", "DDT_GRID_MODE", "DDT_SPREAD", "DDT_XONCE_G", "DDT_XUB_SMALL", "DDT_SELF_VIA_DIRECT", "DDT_FORCE_SYS_SCOPE"):
            os.environ.pop(k, None)
        env = dict(VARIANTS[n])
        mode = env.pop("_mode", "p2p")
        os.environ.update(env)
        ddt.reload_env()
        c = ddt.Comm.single(0)
        if cfg == "cfg1":
            wls[n] = bench.HaloWorkload(ddt, torch, 0, 1, (128, 128, 128), FACE_DIRS, 1, mode, c, 2,
                                        replicas=int(os.environ.get("R", "96")), graph=False)
        else:
            wls[n] = bench.HaloWorkload(ddt, torch, 0, 1, (512, 512, 512), ALL_DIRS, 4, mode, c, 4, replicas=1,
                                        graph=False)
    os.environ.clear()
    os.environ.update(base_env)
    ddt.reload_env()
    return wls


def main():
    which = sys.argv[1] if len(sys.argv) > 1 else "all"
    names = os.environ.get("VARIANTS", ",".join(VARIANTS)).split(",")
    torch.cuda.set_device(0)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    out = {}
    for cfg in (["cfg1", "comb"] if which == "all" else [which]):
        wls = build(cfg, names)
        K = 200 if cfg == "cfg1" else 40
        res = {n: [] for n in names}
        for _ in range(int(os.environ.get("ROUNDS", "5"))):
            for n in names:
                ms, _ = bench.run_steps(torch, wls[n], K, 5, False, None, capture=True, flush_buf=flush)
                res[n].append(ms * 1e3)
        out[cfg] = {n: {"median_us": round(statistics.median(v), 3), "min_us": round(min(v), 3)} for n, v in
                    res.items()}
        d = out[cfg]["direct"]["median_us"] if "direct" in out[cfg] else None
        if d:
            for n in names:
                out[cfg][n]["vs_direct"] = round(out[cfg][n]["median_us"] / d, 3)
        print(cfg, json.dumps(out[cfg]), flush=True)
        for w in wls.values():
            w.close()
        del wls
        torch.cuda.empty_cache()
    return out


if __name__ == "__main__":
    main()
