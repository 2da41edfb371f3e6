python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
GP_DEBUG=1 timeout 300 python -u scripts/trace_levels.py C4 2>&1 | grep -E "level|rep" | grep -v "enqueue\|reported" | tail -12 | cut -c1-600
python - <<'PY'
import sys, torch
sys.path.insert(0,'.')
import graphgen as G
g = G.make_config("C4", device="cuda")
adjp = g["adjp"].long()
deg = (adjp[1:] - adjp[:-1])
n = deg.numel()
print("n", n, "nnz", int(adjp[-1]), "max deg", int(deg.max()), "rows >4096", int((deg > 4096).sum()), "arcs in them", int(deg[deg > 4096].sum()), "rows>256", int((deg>256).sum()), "isolated", int((deg==0).sum()))
PY
