"""TMA issue rate: single-thread vs whole-warp (elect inside the asm) producer loops."""
import sys, json, ctypes, torch
sys.path.insert(0, "/root/repo")
exec(open("/root/repo/scratch/tma_micro.py").read().split("for box in")[0])
for box in (16, 64, 128):
    for ctas in (1, 148):
        for stages in (4, 8):
            for same in (0, 2):
                print(json.dumps(run(box, ctas, stages, same)), flush=True)
