import sys
sys.path.insert(0, ".")
import ctypes as C
import torch
from paper_conf_eurosys_wulywdyfwwj26_b200 import grouter as G
lib = G.load()
s = torch.cuda.Stream()
names = {0: "<<<>>> int arg", 1: "<<<>>> SmallParams", 2: "<<<>>> CopyParams (5 KB)", 3: "LaunchKernelEx PDL",
         4: "LaunchKernelEx", 5: "EventRecord", 6: "EventQuery", 7: "launch_copy 4 KiB (wv8)",
         8: "launch_copy 38.5 MB (wv8)", 9: "event record + launch_copy 38.5 MB",
         10: "driver cuLaunchKernelEx PDL SmallParams", 11: "driver cuLaunchKernelEx SmallParams"}
for mode, off in (("back-to-back", 0), ("idle stream (sync before each)", 100)):
    for stream_name, st in (("torch stream", s.cuda_stream), ("legacy default", 0)):
        for kind in (0, 1, 2, 3, 4, 5, 6, 7, 8, 9, 10, 11):
            for blocks in ((1, 592) if kind < 7 or kind >= 10 else (0,)):
                v = C.c_double(0)
                for rep in range(2):
                    G.check(lib.grouter_test_launch_cost(kind + off, 500, blocks, st or None, C.byref(v)))
                print(mode, stream_name, names[kind], "blocks", blocks, "us/call", round(v.value, 2), flush=True)
