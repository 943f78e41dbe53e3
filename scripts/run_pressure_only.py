import sys, json; sys.path.insert(0, '.')
import bench, paper_conf_isca_fenghzly025_b200 as wk
print(json.dumps(bench.run_pressure(wk, 0)))
