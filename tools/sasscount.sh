# per-kernel SASS size and selected mnemonics: bash tools/sasscount.sh <lib.so> <kernel regex>
cuobjdump -sass "$1" 2>/dev/null | awk -v re="$2" '
/Function :/ { inside = ($0 ~ re); if (inside) { name=$3; n=0; c=0; cas=0; red=0; shfl=0 } next }
inside && /^        \/\*[0-9a-f]+\*\// { n++; if ($0 ~ /CgaCtaId/) c++; if ($0 ~ /ATOMS.CAST/) cas++; if ($0 ~ /REDG/) red++; if ($0 ~ /SHFL/) shfl++ }
inside && /\.\.\.\.\.\.\.\.\.\./ { print name, "instr", n, "CgaCtaId", c, "ATOMS.CAST", cas, "REDG", red, "SHFL", shfl; inside=0 }'
