"""Runs the README Python snippet (documentation check, GPU box)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.chdir(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import re
src = open("README.md").read()
blocks = re.findall(r"```python\n(.*?)```", src, re.S)
code = blocks[0]
print(code)
exec(compile(code, "readme", "exec"))
print("summary", summary["best_cost"], "greedy", gres["dag_cost"])
_, s2 = run2.extract(); print("converge run best", s2["best_cost"])
print("learned W1", learned.mlp["W1"].shape)
