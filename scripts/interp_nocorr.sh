python scripts/interp_nocorr.py 512
SF_LIB=dbg/libsf_nocorr.so python scripts/interp_nocorr.py 512
python scripts/interp_nocorr.py 512
SF_LIB=dbg/libsf_nocorr.so python scripts/interp_nocorr.py 512
