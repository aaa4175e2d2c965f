for c in 0 1 2; do for ef in 0 1; do
  if [ $ef = 0 ]; then export RGSQR_K2_NO_EF=1; else unset RGSQR_K2_NO_EF; fi
  echo "chol $c ef $ef $(RGSQR_LEAF_CHOL=$c python bench.py --no-qrsvd --steps 20 2>/dev/null | grep -o '"ms_per_step": [0-9.]*' | head -1)"
done; done
