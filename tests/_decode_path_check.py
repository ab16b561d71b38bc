"""Run by test_gpu_linear.test_decode_forced_path in a subprocess with SQ_GEMV_PATH=mma|tc (the
path choice is read once per process): decode parity of the forced kernel against the oracle."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
from oracle import oracle as O
import paper_conf_cluster_zhaowplw25_b200 as sq


def main():
    worst = 0.0
    for bits in (3, 4, 8, 16):
        for (n, k) in ((256, 512), (768, 768), (384, 1152), (9600, 256)):
            w = synth.weight_f16(900 + n + bits, n, k)
            b = synth.bias_f16(901 + n, n)
            qo = O.QWeight(w, bits, bias=b)
            qg = sq.QLinear.from_fp16(torch.from_numpy(w).cuda(), bits, torch.from_numpy(b).cuda())
            for m in (1, 3, 5, 8, 9, 16, 32):
                x = synth.act_f16(902 + m, m, k)
                ref = O.linear(x, qo)
                y = torch.empty((m, n), dtype=torch.float16, device="cuda")
                sq.sq_linear_decode(qg, torch.from_numpy(x).cuda(), y, 0)
                torch.cuda.synchronize()
                yy = y.float().cpu().numpy().astype(np.float64)
                err = float(np.abs(yy - ref).max() / np.abs(ref).max())
                worst = max(worst, err)
                assert err <= 2e-3, (os.environ.get("SQ_GEMV_PATH"), bits, n, k, m, err)
                if bits != 16 and m <= 16:
                    # group sums supplied by the caller (sq_xsum) instead of computed in the kernel
                    xd = torch.from_numpy(x).cuda()
                    y2 = torch.empty_like(y)
                    sq.sq_linear_decode(qg, xd, y2, 0, xsum=sq.sq_xsum(xd))
                    torch.cuda.synchronize()
                    err = float(np.abs(y2.float().cpu().numpy().astype(np.float64) - ref).max() / np.abs(ref).max())
                    worst = max(worst, err)
                    assert err <= 2e-3, (os.environ.get("SQ_GEMV_PATH"), "xsum", bits, n, k, m, err)
                # fp32-residual epilogue (o / fc2): y_f32 += x W~^T + bias
                y0 = synth.act_f16(903 + m, m, n).astype(np.float32)
                ya = torch.from_numpy(y0.copy()).cuda()
                sq.sq_linear_decode(qg, torch.from_numpy(x).cuda(), ya, sq.SQ_EPI_F32_ACCUM)
                torch.cuda.synchronize()
                dy = ya.cpu().numpy().astype(np.float64) - y0.astype(np.float64)
                err = float(np.abs(dy - ref).max() / np.abs(ref).max())
                worst = max(worst, err)
                assert err <= 2e-3, (os.environ.get("SQ_GEMV_PATH"), "accum", bits, n, k, m, err)
    # adversarial groups (R20: +-65504 spans saturate; constant, -0, subnormal, ties) on the forced kernel
    for bits in (3, 4, 8):
        n, k = 256, 512
        w = synth.adversarial_weight_f16(60 + bits, n, k)
        qo = O.QWeight(w, bits)
        qg = sq.QLinear.from_fp16(torch.from_numpy(w).cuda(), bits)
        keep = np.setdiff1d(np.arange(n), [3, 8, 9, 10, 11, 12])
        for m in (1, 5, 32):
            x = synth.act_f16(904 + m, m, k)
            ref = O.linear(x, qo)
            y0 = np.zeros((m, n), np.float32)
            ya = torch.from_numpy(y0).cuda()
            sq.sq_linear_decode(qg, torch.from_numpy(x).cuda(), ya, sq.SQ_EPI_F32_ACCUM)
            torch.cuda.synchronize()
            yy = ya.cpu().numpy().astype(np.float64)
            assert np.isfinite(yy).all(), ("adv", bits, m)
            for cols in (slice(None), keep):
                err = float(np.abs(yy[:, cols] - ref[:, cols]).max() / np.abs(ref[:, cols]).max())
                worst = max(worst, err)
                assert err <= 2e-3, (os.environ.get("SQ_GEMV_PATH"), "adv", bits, m, err)
    print("ok worst", worst)


def full(bits):
    """configs[1] OPT-13B fc1 at m = 1 on the forced kernel; sampled rows vs the oracle."""
    n, k, m = 20480, 5120, 1
    seed = synth.weight_seed(1, "fc1")
    wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
    synth.device_weight_f16(wd.data_ptr(), seed, n, k)
    qg = sq.QLinear.from_fp16(wd, bits)
    del wd
    x = synth.act_f16(17, m, k)
    y = torch.empty((m, n), dtype=torch.float16, device="cuda")
    sq.sq_linear_decode(qg, torch.from_numpy(x).cuda(), y, 0)
    torch.cuda.synchronize()
    yy = y.float().cpu().numpy().astype(np.float64)
    rows = np.random.default_rng(bits).choice(n, 64, replace=False)
    rows[0], rows[1] = 0, n - 1
    ref = O.linear(x, O.QWeight(synth.weight_f16(seed, n, k, rows=rows), bits))
    err = float(np.abs(yy[:, rows] - ref).max() / np.abs(ref).max())
    assert err <= 2e-3, ("full", os.environ.get("SQ_GEMV_PATH"), bits, err)
    # determinism of the cross-CTA fix-up at the full grid
    y2 = torch.empty_like(y)
    sq.sq_linear_decode(qg, torch.from_numpy(x).cuda(), y2, 0)
    torch.cuda.synchronize()
    assert torch.equal(y, y2)
    print("ok full", bits, err)


def bloom(bits):
    """configs[4] BLOOM-176B linears at their full size (fc1 57344 x 14336, fc2 14336 x 57344) on the
    automatic decode path (K2s at m = 1 / 8, K2c at m = 32): sampled rows vs the oracle, bitwise repeat."""
    for (n, k, name) in ((57344, 14336, "fc1"), (14336, 57344, "fc2")):
        seed = synth.weight_seed(3, name)
        wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
        synth.device_weight_f16(wd.data_ptr(), seed, n, k)
        qg = sq.QLinear.from_fp16(wd, bits)
        del wd
        rows = np.random.default_rng(bits + n).choice(n, 32, replace=False)
        rows[0], rows[1] = 0, n - 1
        qo = O.QWeight(synth.weight_f16(seed, n, k, rows=rows), bits)
        for m in (1, 8, 32):
            x = synth.act_f16(31 + m, m, k)
            xd = torch.from_numpy(x).cuda()
            y = torch.empty((m, n), dtype=torch.float16, device="cuda")
            sq.sq_linear_decode(qg, xd, y, 0)
            y2 = torch.empty_like(y)
            sq.sq_linear_decode(qg, xd, y2, 0)
            torch.cuda.synchronize()
            assert torch.equal(y, y2), ("bloom repeat", name, bits, m)
            ref = O.linear(x, qo)
            yy = y.float().cpu().numpy().astype(np.float64)[:, rows]
            err = float(np.abs(yy - ref).max() / np.abs(ref).max())
            assert err <= 2e-3, ("bloom", name, bits, m, err)
        del qg
        torch.cuda.empty_cache()
    print("ok bloom", bits)


def canary():
    """Out-of-bounds guard for the forced kernel (compute-sanitizer is closed on this pool): y is a
    strided window of a larger buffer pre-filled with a sentinel, the workspace is followed by a
    sentinel pad; after two launches every sentinel byte is intact, every split-k counter has reset
    to 0 and the window matches the oracle."""
    SENT = 0x7C01  # an fp16 NaN payload no kernel writes
    for bits in (3, 4, 8):
        for (n, k) in ((2048, 1536), (256, 4608), (9600, 256)):
            w = synth.weight_f16(910 + n + bits, n, k)
            qo = O.QWeight(w, bits)
            qg = sq.QLinear.from_fp16(torch.from_numpy(w).cuda(), bits)
            for m in (1, 5, 8):
                x = synth.act_f16(911 + m, m, k)
                ref = O.linear(x, qo)
                big = torch.full((m + 2, n + 64), SENT, dtype=torch.int16, device="cuda").view(torch.float16)
                y = big[1:m + 1, 32:32 + n]
                nws = sq.sq_linear_workspace_bytes(qg, m)
                wsb = torch.zeros(nws + 4096, dtype=torch.uint8, device="cuda")
                wsb[nws:] = 0xA5
                for _ in range(2):
                    sq.sq_linear_decode(qg, torch.from_numpy(x).cuda(), y, 0, ws=wsb[:nws])
                torch.cuda.synchronize()
                raw = big.view(torch.int16).cpu().numpy()
                mask = np.ones(raw.shape, bool)
                mask[1:m + 1, 32:32 + n] = False
                assert (raw[mask] == SENT).all(), ("canary y", bits, n, k, m)
                assert (wsb[nws:].cpu().numpy() == 0xA5).all(), ("canary ws", bits, n, k, m)
                cnt = wsb[:(65536 // 16) * 4].view(torch.int32).cpu().numpy()
                assert (cnt == 0).all(), ("counters not reset", bits, n, k, m)
                yy = y.float().cpu().numpy().astype(np.float64)
                err = float(np.abs(yy - ref).max() / np.abs(ref).max())
                assert err <= 2e-3, ("canary parity", bits, n, k, m, err)
    print("ok canary")


if __name__ == "__main__":
    if len(sys.argv) > 2 and sys.argv[1] == "full":
        full(int(sys.argv[2]))
    elif len(sys.argv) > 1 and sys.argv[1] == "canary":
        canary()
    elif len(sys.argv) > 2 and sys.argv[1] == "bloom":
        bloom(int(sys.argv[2]))
    else:
        main()
