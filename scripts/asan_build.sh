#!/bin/bash
# Host-side AddressSanitizer + UndefinedBehaviorSanitizer build of libcrsd (the
# builder, C-ABI, planner, JIT generator) and of the oracle's C code, then the
# CPU test suites that exercise them (host-only handles, no GPU needed).
# Output: profiles/r02/sanitize/asan_ubsan_cpu.txt
set -e
cd "${GRAFT_REPO_ROOT:-/root/repo}"
B=/tmp/crsd_asan
mkdir -p $B
NV=/usr/local/cuda/bin/nvcc
INC=$(python -c "import sys; sys.path.insert(0,'paper_conf_icpp_sunzwzyr11_b200'); import _build; print(_build._nccl_dirs()[0])")
LIBD=$(python -c "import sys; sys.path.insert(0,'paper_conf_icpp_sunzwzyr11_b200'); import _build; print(_build._nccl_dirs()[1])")
SAN="-fsanitize=address,undefined -fno-omit-frame-pointer -fno-sanitize-recover=undefined"
XSAN="-Xcompiler -fsanitize=address -Xcompiler -fsanitize=undefined -Xcompiler -fno-omit-frame-pointer -Xcompiler -fno-sanitize-recover=undefined"
objs=""
for f in paper_conf_icpp_sunzwzyr11_b200/csrc/*.cpp; do
  o=$B/$(basename $f).o
  $NV -O1 -g -std=c++17 -Xcompiler -fPIC,-fopenmp $XSAN -I$INC -Iinclude -gencode arch=compute_100a,code=sm_100a -c $f -o $o
  objs="$objs $o"
done
for f in paper_conf_icpp_sunzwzyr11_b200/csrc/*.cu; do
  o=$B/$(basename $f).o
  $NV -O3 -std=c++17 -Xcompiler -fPIC -I$INC -Iinclude -gencode arch=compute_100a,code=sm_100a -c $f -o $o
  objs="$objs $o"
done
$NV -shared -gencode arch=compute_100a,code=sm_100a -o $B/libcrsd.so $objs -L$LIBD -l:libnccl.so.2 -Xlinker -rpath,$LIBD -lgomp -ldl $XSAN
gcc -O1 -g -ffp-contract=off $SAN -fPIC -shared -o $B/liboracle.so oracle/coo_spmv.c -lm
gcc -O1 -g -ffp-contract=off $SAN -fopenmp -fPIC -shared -o $B/liboracle_native.so oracle/coo_native.c
echo built
# run the CPU suites against the sanitized libraries in a scratch copy of the repo
R=/tmp/crsd_asan_repo
rm -rf $R && mkdir -p $R && tar --exclude=.git --exclude=gpurun_out -cf - . | tar -xf - -C $R
cp $B/libcrsd.so $R/paper_conf_icpp_sunzwzyr11_b200/libcrsd.so
cp $B/liboracle.so $R/oracle/liboracle.so
cp $B/liboracle_native.so $R/oracle/liboracle_native.so
touch $R/paper_conf_icpp_sunzwzyr11_b200/libcrsd.so $R/oracle/*.so
ASAN_LIB=$(gcc -print-file-name=libasan.so)
UBSAN_LIB=$(gcc -print-file-name=libubsan.so)
cd $R
LD_PRELOAD="$ASAN_LIB $UBSAN_LIB" ASAN_OPTIONS=detect_leaks=0,protect_shadow_gap=0,halt_on_error=1 UBSAN_OPTIONS=print_stacktrace=1,halt_on_error=1 \
  timeout 3000 python -m pytest tests/test_builder.py tests/test_oracle_pins.py tests/test_dist_gloo.py tests/test_gen.py -q -m "not gpu" \
  -p no:cacheprovider -k "not codelets_compile" 2>&1 | tail -4
# (the deselected test runs nvcc as a subprocess, which inherits LD_PRELOAD);
# the JIT generator and the in-process NVRTC compile under the sanitizers:
LD_PRELOAD="$ASAN_LIB $UBSAN_LIB" ASAN_OPTIONS=detect_leaks=0,protect_shadow_gap=0,halt_on_error=1 UBSAN_OPTIONS=print_stacktrace=1,halt_on_error=1 \
  timeout 1200 python - <<'PY'
import numpy as np, gen
from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix
for name, a in [("c1", gen.config1()), ("c3s", gen.config3(n=24)), ("rand", gen.random_diagonal(3000, 3000, 3, ndiag=8, max_off=400, n_scatter=40))]:
    for dt in (np.float64, np.float32):
        A = CRSDMatrix.from_coo(a.nrows, a.ncols, a.row, a.col, a.val.astype(dt), host_only=True, variant=4)
        src, cub = A.jit_source(), A.jit_cubin()
        print(f"jit {name} {np.dtype(dt).name}: source {len(src)} B, cubin {len(cub)} B")
PY
