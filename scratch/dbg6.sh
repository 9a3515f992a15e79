for v in O0 O1 O2; do PHMM_LIB=scratch/variants/libphmm_$v.so python scratch/dbg6.py; done
