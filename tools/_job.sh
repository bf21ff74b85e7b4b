bash tools/gpu.sh h14 build
ab() { tag=$1; shift; env "$@" timeout 300 python tools/ab_step.py --tag $tag 2>/dev/null | tee -a gpurun_out/h14_ab.jsonl | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['tag'], round(d['us_per_step'],2), round(d['min'],2), round(d['max'],2))"; }
ab nofold ASGD_K0_FOLD=0
ab fold X=1
ab fold_t256 ASGD_K0_THREADS=256
ab fold_t128 ASGD_K0_THREADS=128
ab fold_k3dz_t128 ASGD_K3DZ=1 ASGD_K0_THREADS=128
ab fold_k3dz ASGD_K3DZ=1
ab late ASGD_K0_FOLD=0 ASGD_K0_LATE=1
ab fold_onepass ASGD_ONEPASS=1
ab fold_tma ASGD_K1_TMA=1
ab nofold_c32 ASGD_K0_FOLD=0 ASGD_K0_CTAS=32 ASGD_K0_THREADS=256 ASGD_K1_CTAS=264
ab fold_g2fuse ASGD_G2_FUSE=1
ab fold_nopdl ASGD_PDL=0
