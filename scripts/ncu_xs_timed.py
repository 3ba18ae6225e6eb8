"""The headline launch exactly as bench.py times it, for ncu: B200 layouts, L2 set-aside at
the device maximum, persisting lines reset + L2 flushed, then ONE omprt_xs_flat_rt launch
over the 17M lookups with its access-policy window (argv[1] == "nowin": without it;
"stream": the same window set as a STREAM attribute through cuda-python and the launch
without its own -- ncu drops the launch attribute, profiles/README.md).
  ncu ... python scripts/ncu_xs_timed.py [win|nowin|stream] [reps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    mode = sys.argv[1] if len(sys.argv) > 1 else "win"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    dev = torch.device("cuda", 0)
    t = gen.XSTables(**gen.XS_SMALL)
    d = omprt.XSDeviceTables(t, dev, accel=True)
    n = 17_000_000
    ver = torch.zeros(n, dtype=torch.uint64, device=dev)
    scrub = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    got = omprt.omprt_l2_set_aside(1 << 40)
    F = omprt.OMPRT_XS_FLAT | (omprt.OMPRT_XS_NO_L2_PERSIST if mode != "win" else 0)
    s = torch.cuda.current_stream()
    if mode == "stream":
        from cuda.bindings import runtime as rt
        dev_id = 0
        err, maxwin = rt.cudaDeviceGetAttribute(
            rt.cudaDeviceAttr.cudaDevAttrMaxAccessPolicyWindowSize, dev_id)
        val = rt.cudaStreamAttrValue()
        w = val.accessPolicyWindow
        nbytes = min(d._pack.numel(), maxwin)
        w.base_ptr = d._pack.data_ptr()
        w.num_bytes = nbytes
        w.hitRatio = min(1.0, got / nbytes)
        w.hitProp = rt.cudaAccessProperty.cudaAccessPropertyPersisting
        w.missProp = rt.cudaAccessProperty.cudaAccessPropertyStreaming
        err, = rt.cudaStreamSetAttribute(s.cuda_stream,
                                         rt.cudaStreamAttrID.cudaLaunchAttributeAccessPolicyWindow,
                                         val)
        print("stream window", err, nbytes, w.hitRatio, flush=True)
    for _ in range(reps):
        torch.cuda.synchronize()
        omprt.omprt_l2_reset_persisting()
        scrub.fill_(1.0)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        omprt.omprt_xs_lookup(d, gen.XS_LOOKUP_SEED, 0, n, ver, None, 0, 256, F)
        b.record(s)
        torch.cuda.synchronize()
        print(f"{mode} set_aside={got} event_ms={a.elapsed_time(b):.4f}", flush=True)


if __name__ == "__main__":
    main()
