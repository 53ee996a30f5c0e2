# parity tests of a compile-time variant: GDROID_NVCC_FLAGS="<flags>" bash scripts/gpu_flags_test.sh
python -c "import paper_conf_ipps_yuwobby20_b200._build as b; b.build()" || exit 1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
