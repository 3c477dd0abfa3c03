# Build A/B variants of libmst.so: VARS="name:-DFLAG=1 -DX name2:" bash tools/abvar.sh
# -> build/ab/<name>.so (run them with MST_LIB=build/ab/<name>.so, tools/abrun2.sh)
mkdir -p build/ab
for v in $VARS; do
  name=${v%%:*}; flags=${v#*:}
  MST_NVCC_FLAGS="$flags" python - "$name" <<'PY'
import os, sys, shutil
from paper_conf_ppopp_nasrebp13_b200 import _build
out = os.path.join(_build.ROOT, "build", "ab", sys.argv[1] + ".so")
_build.LIB = out
_build.build(force=True)
print("built", out, os.environ.get("MST_NVCC_FLAGS"))
PY
done
