bash tools/ab.sh "--steps 100 --cmap-t 128 --cmap-t1 32" variants/libam_l08k_t32.so
bash tools/ab.sh "--steps 100 --cmap-t 128 --cmap-t1 24" variants/libam_l08k_t24.so
bash tools/ab.sh "--steps 100 --cmap-t 128 --cmap-t1 48" variants/libam_l04k_t48.so variants/libam_l016k_t48.so
bash tools/ab.sh "--steps 100 --cmap-t 144 --cmap-t1 48" variants/libam_l08k_t48_t144.so
