/* The single SASS-only code object holding the whole kernel catalog,
 * embedded in .rodata of libpask.so and handed to cuLibraryLoadData. */
        .section .rodata.pask_fatbin,"a",@progbits
        .balign 64
        .globl pask_fatbin_start
        .hidden pask_fatbin_start
pask_fatbin_start:
        .incbin PASK_FATBIN_PATH
        .globl pask_fatbin_end
        .hidden pask_fatbin_end
pask_fatbin_end:
        .byte 0
        .section .note.GNU-stack,"",@progbits
