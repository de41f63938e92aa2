# build libglb.so of git revision $1 into build/ab/libglb_$1.so (for GLB_LIBRARY A/B runs)
set -e
REV=$1
D=$(mktemp -d)
git archive $REV paper_conf_eurosys_yangtswycyz22_b200/csrc include | tar -x -C $D
mkdir -p build/ab
for f in $D/paper_conf_eurosys_yangtswycyz22_b200/csrc/*.cu; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -I$D/include --expt-relaxed-constexpr -c $f -o $D/$(basename $f .cu).o &
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o build/ab/libglb_$REV.so $D/*.o -lcudart
rm -rf $D
echo build/ab/libglb_$REV.so
