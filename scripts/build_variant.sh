# usage: bash scripts/build_variant.sh NAME "-DFOO=1 ..."  -> variants/libsmoothe_NAME.so
# (A/B experiments with scripts/ab_exp.sh; variants/ is git-ignored but travels to the GPU box)
set -e
# SRC=<dir holding csrc/ and ../include> builds another tree (e.g. a git worktree)
OUT=$(cd "$(dirname "$0")/.." && pwd)/variants
cd "${SRC:-$(dirname "$0")/../paper_conf_asplos_caiydyz25_b200}"
NAME=$1; DEFS=$2
B=/tmp/smoothe_variant_$NAME; rm -rf $B; mkdir -p $B $OUT
ARCH="-gencode arch=compute_100a,code=sm_100a"
for f in csrc/*.cu; do
  nvcc -std=c++17 -O3 -lineinfo $ARCH -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -Icsrc $DEFS -c $f -o $B/$(basename $f .cu).o &
done
for f in csrc/*.cpp; do g++ -std=c++17 -O3 -fPIC -fvisibility=hidden -I/usr/local/cuda/include -Icsrc $DEFS -c $f -o $B/$(basename $f .cpp).o & done
wait
nvcc $ARCH -shared -cudart static -o $OUT/libsmoothe_$NAME.so $B/*.o
echo built $OUT/libsmoothe_$NAME.so
