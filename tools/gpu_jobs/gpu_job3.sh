cd $GRAFT_REPO_ROOT
timeout 900 python tools/debug_variants.py 20,34,70 > gpurun_out/debug_variants.jsonl 2>&1
cat > /tmp/one.py <<'PY'
import sys; sys.path.insert(0, "tests"); sys.path.insert(0, ".")
from cases import make_case, run_gpu, check
case = make_case("jacobi7", (20, 34, 70))
g, p = run_gpu("jacobi7", (20, 34, 70), case)
print(check("jacobi7", (20, 34, 70), g, case))
PY
timeout 300 compute-sanitizer --tool memcheck python /tmp/one.py > gpurun_out/sanitizer.log 2>&1
echo done > gpurun_out/done.txt
