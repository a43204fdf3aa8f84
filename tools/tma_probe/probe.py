import ctypes, sys, os
use_torch = sys.argv[1] == "torch"
if use_torch:
    import torch
    torch.zeros(1, device="cuda")
L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libprobe.so"))
L.probe_main(int(sys.argv[2]))
