import json, sys
for l in open(sys.argv[1]):
    d = json.loads(l)
    print(d["batch"], round(d["astra"]), round(d["cudnn"]), round(d["astra_over_cudnn"], 2), d["explore_steps"], d["variants"][-1])
