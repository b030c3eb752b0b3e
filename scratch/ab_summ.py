import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
r = d["regions_ms"]
print(round(d["value"]), round(r["bptt_chain_ms"], 3), round(r["fwd_chain_ms"], 3), d["clocks"]["sm_mhz"], d["tuner"]["variant"])
